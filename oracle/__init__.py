"""VPPS oracle — TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU (NumPy float64) implementation of what the VPPS hot
path computes (§III).  Only tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / --impl reference legs may import anything from here.  The product
path (paper_conf_micro_khorasanieas18_b200/) never imports it and shares no code with it.

Modules
  models.py  — cell-level forward and hand-written reverse pass of M1 (LSTM), M2 (BiLSTM
               tagger), M3 (child-sum Tree-LSTM), M4 (binary Tree-LSTM); summed loss (L205);
               fused SGD update (L129, L197).  Pinned by tests/test_oracle_models.py.
  plan.py    — weight-matrix distribution: the paper's round-robin dealer (L92, Fig.4,
               Eq.(1), fn6 L127, L106/L241) and the B200 unit-bundle plan of
               SPEC_SCRIPT.md §P.  Pinned by paper values in tests/test_oracle_plan.py.
  script.py  — level sort, scheduling, signal/wait placement, pool plan and word encoding of
               SPEC_SCRIPT.md §S/§E (L139-169).  Pinned by the Fig.6(d) S/W pattern, the
               L159/L169 sizes and structural invariants; the exact words are
               "parity unpinned" by the paper beyond that and are checked
               bit-exactly against the independent C++ implementation.
"""
