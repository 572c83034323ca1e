"""Per-tensor gradient errors of the chain cells against the oracle (debug aid):
    python tools/chain_debug.py"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402

import synth  # noqa: E402
import test_gpu_parity as t  # noqa: E402
from oracle import models as M  # noqa: E402

for cell, H, batch, lens in [("lstm", 32, 3, (1, 6)), ("lstm", 64, 3, (1, 6)), ("lstm", 128, 3, (1, 6)),
                             ("lstm", 256, 3, (1, 6)), ("lstm", 256, 40, (1, 30)), ("bilstm", 32, 3, (1, 6)),
                             ("bilstm", 64, 3, (1, 6)), ("bilstm", 256, 5, (1, 12)), ("gru", 32, 3, (1, 6)),
                             ("gru", 64, 5, (1, 9)), ("gru", 256, 40, (1, 30))]:
    rng = np.random.default_rng(5)
    if cell in ("lstm", "gru"):
        graphs = [synth.chain(rng, int(rng.integers(lens[0], lens[1] + 1)), 100, lm=True) for _ in range(batch)]
        C, V, kw = 100, 100, {}
    else:
        graphs = synth.tagger_batch(rng, batch, lens, 64, 9)
        C, V, kw = 9, 64, dict(mlp=32)
    m, P, X, loss, params, grads, dX = t.run_case(cell, H, H, C, graphs, V, seed=7, **kw)
    lo, Go, dXo = M.forward_backward(cell, P, X, graphs, H)
    gv = m.views(grads.cpu())
    errs = {n: t.rel(gv[n].numpy(), Go[n]) for n, _ in m.shapes}
    print(cell, H, batch, "loss", abs(loss - lo) / abs(lo), " ".join(f"{k}={v:.1e}" for k, v in errs.items()),
          "dX", f"{t.rel(dX.cpu().numpy(), dXo):.1e}", flush=True)
