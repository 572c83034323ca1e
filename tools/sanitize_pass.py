"""One small training pass per device path, for compute-sanitizer (memcheck / racecheck / synccheck):
    compute-sanitizer --tool memcheck python tools/sanitize_pass.py [dataflow|dataflow128|levelgemm|chain|level|grid]
Exits non-zero if a pass disagrees with the oracle (so a sanitizer-induced change in behaviour shows)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from oracle import models as M  # noqa: E402
from paper_conf_micro_khorasanieas18_b200 import vpps  # noqa: E402


def main(which):
    if which == "dataflow":
        cell, H, C, V, kw = "binary", 256, 5, 64, dict(cluster=16, dataflow=True)
        graphs = synth.tree_batch(np.random.default_rng(1), 3, (2, 12), V, C)
    elif which == "dataflow128":                 # H = 128: groups of 8 CTAs
        cell, H, C, V, kw = "binary", 128, 5, 64, dict(cluster=8, dataflow=True)
        graphs = synth.tree_batch(np.random.default_rng(1), 3, (2, 12), V, C)
    elif which == "levelgemm":                   # level path with the library's own GEMM tiles
        cell, H, C, V, kw = "binary", 64, 5, 64, dict(level=1)
        graphs = synth.tree_batch(np.random.default_rng(1), 3, (2, 12), V, C)
    elif which == "chain":                       # LSTM LM on the chain recurrence
        cell, H, C, V, kw = "lstm", 128, 40, 40, dict(level=1)
        graphs = synth.config_batch("c3", 0, batch=3, V=40, C=40)
    elif which == "grid":
        cell, H, C, V, kw = "binary", 32, 5, 64, {}
        graphs = synth.tree_batch(np.random.default_rng(1), 3, (2, 12), V, C)
    else:
        cell, H, C, V, kw = "bilstm", 32, 9, 64, dict(mlp=16)
        graphs = synth.tagger_batch(np.random.default_rng(2), 3, (1, 8), V, C)
    rng = np.random.default_rng(0)
    shapes = vpps.param_shapes(cell, H, H, C, kw.get("mlp", 256))
    P = synth.init_params(shapes, rng)
    X = synth.input_table(rng, V, H)
    m = vpps.Model(cell, H, H, C, allocator="cuda", **kw)
    params = torch.zeros(m.n_floats, device="cuda")
    grads = torch.zeros_like(params)
    for name, _ in shapes:
        m.views(params)[name].copy_(torch.from_numpy(P[name]).float())
    m.bind(params, grads)
    inputs = torch.from_numpy(X).float().cuda()
    dX = torch.zeros_like(inputs)
    for rep in range(2):                         # second pass: tagged slots reused with a new epoch
        m.fwd_bwd(m.build_script(graphs), inputs, dX)
    loss = m.latest_loss()
    lo, Go, _ = M.forward_backward(cell, P, X, graphs, H)
    ok = abs(loss - lo) <= 1e-4 * abs(lo)
    gv = m.views(grads.cpu())
    for name, _ in shapes:
        ok &= np.abs(gv[name].double().numpy() - Go[name]).max() <= 1e-4 * max(np.abs(Go[name]).max(), 1e-30)
    print(f"{which}: loss {loss:.6f} oracle {lo:.6f} parity {'ok' if ok else 'FAIL'}")
    sys.exit(0 if ok else 1)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "dataflow")
