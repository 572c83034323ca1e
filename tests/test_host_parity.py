"""Bit-exact parity of the C++ host library (libvpps.so, plan-only mode: no GPU needed) with the
independent Python implementation in oracle/ of SPEC_SCRIPT.md (partition table, script words,
pool plan), plus the C-ABI export check against include/vpps.h."""
import ctypes
import os
import re

import numpy as np
import pytest

import synth
from oracle import models as M
from oracle import plan as oplan
from oracle import script as oscript

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def vpps():
    from paper_conf_micro_khorasanieas18_b200 import vpps as v
    return v


def test_abi_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "vpps.h")).read()
    names = set(re.findall(r"\b(vpps_[a-z_]+)\s*\(", hdr))
    assert len(names) >= 20
    lib = ctypes.CDLL(os.path.join(ROOT, "paper_conf_micro_khorasanieas18_b200", "libvpps.so"))
    for n in sorted(names):
        assert hasattr(lib, n), n


def test_param_shapes_agree_with_oracle(vpps):
    for cell in ("lstm", "binary", "childsum", "gru", "rvnn", "tdlstm"):
        a = [(n, tuple(s)) for n, s in vpps.param_shapes(cell, 8, 4, 3)]
        b = [(n, tuple(s)) for n, s in M.param_shapes(cell, 8, 4, 3)]
        assert a == b


@pytest.mark.parametrize("rows_a", [9, 16, 40])
@pytest.mark.parametrize("pack", [0, 1])
def test_paper_deal_bit_exact(vpps, rows_a, pack):
    mats = [(rows_a, 128), (24, 96), (5, 256)]
    for grads in (0, 1):
        c_rows, c_slots = vpps.paper_deal(mats, 4, 128, 2, pack, grads)
        o_rows, o_slots = oplan.paper_deal(mats, 4, 128, 2, bool(pack), bool(grads))
        assert c_slots == o_slots
        assert np.array_equal(c_rows, np.array(o_rows, dtype=np.int32))


def test_paper_choose_cps_bit_exact(vpps):
    for H in (128, 256, 384, 512):
        mats = [s for (_, s) in M.param_shapes("binary", H, 128, 5) if len(s) == 2]
        for n_sm in (80, 148):
            assert vpps.paper_choose_cps(mats, n_sm) == oplan.choose_cps(mats, n_sm)
    mats = [s for (_, s) in M.param_shapes("binary", 256, 128, 5) if len(s) == 2]
    assert vpps.paper_choose_cps(mats, 80) == 2      # L241 via the C++ path too


@pytest.mark.parametrize("cell,H,E,C", [("binary", 256, 256, 5), ("binary", 1024, 1024, 5),
                                        ("lstm", 32, 32, 16), ("childsum", 128, 128, 5), ("lstm", 256, 256, 1000)])
@pytest.mark.parametrize("G", [1, 2, 4])
def test_partition_table_bit_exact(vpps, cell, H, E, C, G):
    try:
        ref = oplan.unit_plan(cell, H, E, C, n_sm=148, G=G)
    except ValueError:
        with pytest.raises(vpps.VppsError) as e:
            vpps.Model(cell, H, E, C, n_sm=148, groups=G, plan_only=True)
        assert e.value.status == -2
        return
    m = vpps.Model(cell, H, E, C, n_sm=148, groups=G, plan_only=True)
    info = m.plan_info()
    assert (info["n_g"], info["n_act"], info["umax"]) == (ref["n_g"], ref["n_act"], ref["umax"])
    assert np.array_equal(m.partition_table(), np.array(ref["table"], dtype=np.int32))


def _batches(cell, rng, n):
    out = []
    for _ in range(n):
        b = int(rng.integers(1, 9))
        if cell == "lstm":
            out.append([synth.chain(rng, int(rng.integers(1, 12)), 7) for _ in range(b)])
        elif cell == "binary":
            out.append(synth.tree_batch(rng, b, (1, 20), 50, 5))
        else:
            gs = synth.tree_batch(rng, b, (1, 15), 50, 5)
            # child-sum: vary arity and token presence
            gs.append([((), -1, -1), ((0,), 3, 2), ((), 4, -1), ((), 5, -1), ((1, 2, 3), -1, 1)])
            out.append(gs)
    return out


@pytest.mark.parametrize("cell", ["binary", "lstm", "childsum"])
@pytest.mark.parametrize("G", [1, 2, 4])
def test_script_words_bit_exact(vpps, cell, G):
    H, E, C = 8, 8, 7
    m = vpps.Model(cell, H, E, C, n_sm=16, groups=G, plan_only=True)
    rng = np.random.default_rng(100 + G)
    n_act = m.plan_info()["n_act"]
    for graphs in _batches(cell, rng, 12):
        s = m.build_script(graphs)
        ref = oscript.build(cell, graphs, H, E, C, G=G, n_act=n_act)
        w = s.words()
        assert np.array_equal(w, np.array(ref["words"], dtype=np.uint32))
        info = s.info()
        assert (info["pool_words"], info["zero_words"], info["loss_word"], info["n_barriers"]) == \
            (ref["pool_words"], ref["zero_words"], ref["loss_word"], ref["n_bar"])
        assert info["flops"] == M.flop_count(cell, graphs, H, E, C)


@pytest.mark.parametrize("cell", ["binary", "lstm", "childsum"])
def test_script_words_bit_exact_graph_groups(vpps, cell):
    """SPEC S5g (cluster replicas): whole graphs per group, min-load over graph MACs."""
    H, E, C = 16, 16, 7
    m = vpps.Model(cell, H, E, C, n_sm=7 * 16, groups=7, cluster=16, plan_only=True)
    assert m.plan_info()["n_g"] == 16
    rng = np.random.default_rng(77)
    for graphs in _batches(cell, rng, 10):
        s = m.build_script(graphs)
        ref = oscript.build(cell, graphs, H, E, C, G=7, n_act=m.plan_info()["n_act"], by_graph=True)
        assert np.array_equal(s.words(), np.array(ref["words"], dtype=np.uint32))


def test_graph_groups_keep_graphs_whole():
    graphs = synth.tree_batch(np.random.default_rng(5), 9, (2, 12), 50, 5)
    ref = oscript.build("binary", graphs, 8, 8, 5, G=4, n_act=9, by_graph=True)
    w = ref["words"]
    G = w[0]
    pre = w[2:2 + G + 1]
    base = 2 + G + 1
    owner = {}
    for g in range(G):
        st = w[base + pre[g]: base + pre[g + 1]]
        # every record operand in group g's stream belongs to a graph owned by g
        for x in st:
            if x in ref["rec"]:
                gid = ref["nodes"][ref["rec"].index(x)]["graph"]
                assert owner.setdefault(gid, g) == g


def test_script_words_target_config(vpps):
    """TGT shapes (binary H = E = 256, batch 16 SST-shaped trees) on 148 SMs."""
    m = vpps.Model("binary", 256, 256, 5, n_sm=148, plan_only=True)
    for b in range(3):
        graphs = synth.config_batch("tgt", b)
        s = m.build_script(graphs)
        ref = oscript.build("binary", graphs, 256, 256, 5, G=1, n_act=148)
        assert np.array_equal(s.words(), np.array(ref["words"], dtype=np.uint32))


def test_graph_errors(vpps):
    m = vpps.Model("binary", 8, 8, 3, n_sm=16, plan_only=True)
    with pytest.raises(vpps.VppsError) as e:
        m.build_script([[((), 0, -1), ((0,), -1, 1)]])          # unary internal node (R-26)
    assert e.value.status == -4
    with pytest.raises(vpps.VppsError):
        m.build_script([[((), 0, -1), ((), 1, -1), ((0, 0), -1, 1)]])   # two parents edges to one child
    with pytest.raises(vpps.VppsError):
        m.build_script([[((), 0, 5)]])                            # label out of range
    with pytest.raises(vpps.VppsError):
        vpps.Model("binary", 8, 8, 3, n_sm=16, plan_only=True).build_script([[((1,), 0, -1), ((), 0, -1)]])


@pytest.mark.parametrize("cell", ["binary", "lstm", "childsum", "rvnn"])
def test_empty_batch_is_a_graph_error(vpps, cell):
    """Edge case: a batch without nodes (no graphs, or only empty graphs) is rejected with VPPS_E_GRAPH
    (include/vpps.h) rather than launching a pass with nothing to compute.  (The tagger-script cells,
    bilstm and gru, accept it as a pass with T = 0 tokens: zero loss, zero gradients.)"""
    m = vpps.Model(cell, 8, 8, 3, n_sm=16, plan_only=True)
    for graphs in ([], [[]], [[], []]):
        with pytest.raises(vpps.VppsError) as e:
            m.build_script(graphs)
        assert e.value.status == -4


def test_nofit_and_bad_shapes(vpps):
    with pytest.raises(vpps.VppsError) as e:
        vpps.Model("binary", 4096, 4096, 5, n_sm=148, plan_only=True)
    assert e.value.status == -2


def test_widened_cells_host_side(vpps):
    """The NEXT-3 cells (GRU, RvNN, TD-RNN, TD-LSTM) on the host side: op sets accepted in plan-only mode,
    scripts built, the DAG rule applied only to the TD cells, and the TD-RNN's E == H requirement."""
    rng = np.random.default_rng(5)
    assert vpps.param_shapes("tdrnn", 8, 8, 3) == M.param_shapes("tdrnn", 8, 8, 3)
    gru = vpps.Model("gru", 8, 12, 5, plan_only=True)
    info = gru.build_script([synth.chain(rng, 6, 5), synth.chain(rng, 1, 5)]).info()
    assert info["n_levels"] == 6 and info["flops"] > 0
    rv = vpps.Model("rvnn", 8, 12, 5, plan_only=True)
    rv.build_script(synth.tree_batch(rng, 3, (1, 6), 8, 5))
    dag = synth.td_pyramid(rng, 5, 8, 5)                       # inner nodes with two parents
    td = vpps.Model("tdrnn", 8, 8, 5, plan_only=True)
    assert td.build_script([dag]).info()["n_levels"] == 6           # 5 pyramid levels + the head
    vpps.Model("tdlstm", 8, 8, 5, plan_only=True).build_script([dag])
    with pytest.raises(vpps.VppsError):
        rv.build_script([dag])                                  # shared children only in the TD cells
    with pytest.raises(vpps.VppsError):
        vpps.Model("tdrnn", 8, 12, 5, plan_only=True)           # leaves are the input rows: E == H


@pytest.mark.parametrize("cell", ["bilstm", "gru", "lstm"])
def test_chain_script_flops_equal_oracle_count(vpps, cell):
    """The level path's chain scripts (tagger.cpp) report the oracle's algorithmic FLOP count (SURVEY
    §8(d)), ragged lengths including one-token and empty sentences."""
    H, E, C = 8, 12, 5
    rng = np.random.default_rng(31)
    graphs = synth.tagger_batch(rng, 5, (1, 9), 20, C) + [[]]
    m = vpps.Model(cell, H, E, C, plan_only=True, mlp=6, level=1 if cell == "lstm" else 0)
    info = m.build_script(graphs).info()
    assert info["flops"] == M.flop_count(cell, graphs, H, E, C, M=6)


@pytest.mark.parametrize("G", [1, 3, 9])
@pytest.mark.parametrize("dataflow", [True, False])
def test_device_lowering_bit_exact(vpps, G, dataflow):
    """SPEC_SCRIPT.md §D: the gradient GEMM's node lists and the dataflow program that vpps_df executes
    (batches, entries, slot numbering) are bit-identical to oracle/script.py::device_lowering, on
    SST-shaped batches of 1 / 4 / 16 / 64 trees, degenerate ones (a lone labelled leaf, labels on inner
    nodes) and the bench's TGT batches.  A dataflow model leaves the SPEC words out of the blob and still
    returns them, bit-exact, on request."""
    _lowering_case(vpps, 256, 256, 16, G, dataflow)


def test_device_lowering_bit_exact_h128(vpps):
    """The same at H = 128 (groups of 8 CTAs, 16 groups, E = 128): the lowering does not depend on the
    group size; the kernel derives its slot strides from H."""
    _lowering_case(vpps, 128, 128, 8, 16, True)


def _lowering_case(vpps, H, E, ncl, G, dataflow):
    C = 5
    m = vpps.Model("binary", H, E, C, n_sm=ncl * G, groups=G, cluster=ncl, dataflow=dataflow, plan_only=True)
    rng = np.random.default_rng(200 + G)
    inner = [((), 0, 1), ((), 1, -1), ((0, 1), -1, 3), ((), 2, -1), ((2, 3), -1, 0)]
    batches = [synth.tree_batch(rng, b, (1, 50), 64, C) for b in (1, 4, 16, 64)]
    batches += [[[((), 3, 2)]], [inner, inner], synth.config_batch("tgt", 0), synth.config_batch("tgt", 7)]
    for graphs in batches:
        s = m.build_script(graphs)
        blob, lists_off, df_off = s.blob()
        ref = oscript.build("binary", graphs, H, E, C, G=G, n_act=m.plan_info()["n_act"], by_graph=True)
        low = oscript.device_lowering(ref)
        assert lists_off == (0 if dataflow else len(ref["words"]))
        assert np.array_equal(blob[lists_off:], np.array(low["lists"], dtype=np.uint32))
        assert df_off - lists_off == low["df_off"]
        assert np.array_equal(s.words(), np.array(ref["words"], dtype=np.uint32))    # (lazy when dataflow)
        assert s.info()["n_words"] == len(ref["words"])


@pytest.mark.parametrize("cell,H,batch", [("bilstm", 512, 16), ("bilstm", 256, 70), ("lstm", 256, 64),
                                          ("lstm", 32, 4), ("lstm", 128, 300)])
def test_chain_table_bit_exact(vpps, cell, H, batch):
    """SPEC §L: the sentence table of the register-resident chain recurrence (groups per direction from the
    128-register layout: NCL(H) = ceil(4H^2 / 32768) CTAs, 148 SMs) against oracle/script.py::chain_table,
    ragged lengths incl. empty sentences, up to 300 sentences (several per group)."""
    rng = np.random.default_rng(400 + H + batch)
    graphs = synth.tagger_batch(rng, batch, (1, 60), 50, 5) + [[]]
    m = vpps.Model(cell, H, H, 5 if cell == "bilstm" else 50, plan_only=True, mlp=8, level=1)
    blob, lists_off, _ = m.build_script(graphs).blob()
    ncl = -(-4 * H * H // 32768)
    dirs = 2 if cell == "bilstm" else 1
    ref = oscript.chain_table(graphs, (148 // ncl) // dirs, dirs)
    words = np.asarray(blob, dtype=np.int64)
    if ref is None:
        return
    G = ref[0]
    n = len(ref)
    # the table is the last block of the blob (tagger.cpp appends it after the step lists)
    assert np.array_equal(words[-n:], np.array(ref, dtype=np.int64)), (words[-n:][:8], ref[:8])
    assert words[-n] == G


def test_autotune_picks_the_fastest_candidate(vpps):
    """Profile-guided path choice: every candidate is timed and the fastest kept; candidates
    that this build cannot instantiate are skipped (plan-only models stand in for devices here; the timer is
    injected)."""
    fake = {1: 3.0, 2: 1.5, 4: 2.0}
    cands = [dict(groups=g, plan_only=True) for g in (1, 2, 4)] + [dict(groups=3, n_sm=16, plan_only=True)]
    best, res = vpps.autotune("childsum", 8, 8, 5, [], None, candidates=cands,
                              timer=lambda m, b, x: fake[m.options["groups"]])
    assert best == dict(groups=2, plan_only=True)
    assert min(res.values()) == 1.5
    opts = vpps.candidate_options("binary", 256, 5)
    assert opts[0] == dict(cluster=16, dataflow=True) and dict(level=1) in opts
    assert vpps.candidate_options("gru", 256, 1000) == [dict(chain=0), dict(chain=-1)]


def test_auto_replica_groups(vpps):
    """groups < 0: the grid kernel of the tree cells takes 4 replica groups (SPEC P1: 148 CTAs -> 37 per
    group), every other path one group (the LSTM LM at V = 1000 runs on the chain recurrence)."""
    assert vpps.Model("childsum", 128, 128, 5, groups=-1, plan_only=True).plan_info()["n_g"] == 37
    assert vpps.Model("binary", 256, 256, 5, groups=-1, plan_only=True).plan_info()["n_g"] == 37
    assert vpps.Model("lstm", 256, 256, 1000, groups=-1, plan_only=True).plan_info()["n_g"] == 148
    assert vpps.Model("binary", 256, 256, 5, groups=-1, cluster=16, dataflow=True,
                      plan_only=True).plan_info()["n_g"] == 16


def test_bilstmchar_script_host_side(vpps):
    """BiLSTMwChar scripts (plan-only): the host FLOP count equals the oracle's; spellings are accepted only by
    this cell; character ids and tokens are range-checked (a rare word's token is never read)."""
    H, E, C = 32, 64, 9
    g = synth.char_tagger_batch(np.random.default_rng(7), 5, (1, 12), 64, C, 64, rare_from=8)
    assert sum(len(nd[3]) for s_ in g for nd in s_) > 0
    m = vpps.Model("bilstmchar", H, E, C, plan_only=True, mlp=16)
    info = m.build_script(g).info()
    assert info["flops"] == M.flop_count("bilstmchar", g, H, E, C, M=16)
    plain = [[nd[:3] for nd in s] for s in g]
    assert M.flop_count("bilstmchar", plain, H, E, C, M=16) == M.flop_count("bilstm", plain, H, E, C, M=16)
    with pytest.raises(vpps.VppsError):
        vpps.Model("bilstm", H, E, C, plan_only=True, mlp=16).build_script(g)       # spellings need M9
    with pytest.raises(vpps.VppsError):
        m.build_script([[((), 3, 1, (64,))]])                                          # character id >= Vc
    m.build_script([[((), 10 ** 6, 1, (5,))]])                                         # rare: token unused
