"""Repeat one dataflow parity case and print the ‖·‖∞ error ratio of every tensor per run (intermittent-failure
diagnosis: borderline rounding vs a race)."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import synth  # noqa: E402
from oracle import models as M  # noqa: E402
from test_gpu_parity import run_case, rel  # noqa: E402

b = int(sys.argv[1]) if len(sys.argv) > 1 else 5
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 8
graphs = synth.config_batch("tgt", b)
ref = None
for r in range(reps):
    m, P, X, loss, params, grads, dX = run_case("binary", 256, 256, 5, graphs, 4096, 21 + b, True, cluster=16, dataflow=True)
    if ref is None:
        ref = M.forward_backward("binary", P, X, graphs, 256)
    lo, Go, dXo = ref
    gv = m.views(grads.cpu())
    errs = {name: rel(gv[name].numpy(), Go[name]) for name, _ in m.shapes}
    errs["dX"] = rel(dX.cpu().numpy(), dXo)
    nan = {name: int(np.isnan(gv[name].numpy()).sum()) for name, _ in m.shapes}
    print(f"run {r}: loss {abs(loss - lo) / abs(lo):.2e} " + " ".join(f"{k} {v:.2e}" for k, v in errs.items()),
          "nan", {k: v for k, v in nan.items() if v}, flush=True)
