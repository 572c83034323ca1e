"""Mimic the GPU test order (target dataflow cases, then the epochs test) in one process and print every
mismatch of the epochs procedure with its pass, script and error ratios (intermittent-failure diagnosis)."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import synth  # noqa: E402
from oracle import models as M  # noqa: E402
from test_gpu_parity import run_case, rel, _trees  # noqa: E402
from paper_conf_micro_khorasanieas18_b200 import vpps  # noqa: E402

iters = int(sys.argv[1]) if len(sys.argv) > 1 else 6
pre = int(sys.argv[2]) if len(sys.argv) > 2 else 1
H, C, V = 256, 5, 64
bad = 0
for it in range(iters):
    for b in range(pre):   # preceding cases, as in the test session
        run_case("binary", 256, 256, 5, synth.config_batch("tgt", 5 + b), 4096, 26 + b, True, cluster=16, dataflow=True)
    rng = np.random.default_rng(31)
    shapes = vpps.param_shapes("binary", H, H, C)
    P = synth.init_params(shapes, rng)
    m = vpps.Model("binary", H, H, C, cluster=16, dataflow=True)
    params = torch.zeros(m.n_floats, device="cuda")
    grads = torch.zeros_like(params)
    for name, _ in shapes:
        m.views(params)[name].copy_(torch.from_numpy(P[name]).float())
    m.bind(params, grads)
    X = torch.from_numpy(synth.input_table(rng, V, H)).float().cuda()
    batches = [_trees(40 + i, 6, (2, 30), V, C) for i in range(3)]
    scripts = [m.build_script(bb) for bb in batches]
    refs = [M.forward_backward("binary", P, X.cpu().double().numpy(), bb, H) for bb in batches]
    for rep in range(3):
        for k, s in enumerate(scripts):
            m.fwd_bwd(s, X)
            loss = m.latest_loss()
            lo, Go, _ = refs[k]
            gv = m.views(grads.cpu())
            errs = {name: rel(gv[name].numpy(), Go[name]) for name, _ in m.shapes}
            le = abs(loss - lo) / abs(lo)
            if le > 1e-4 or max(errs.values()) > 1e-4:
                bad += 1
                print(f"it {it} rep {rep} script {k} pass {m._passes if hasattr(m, '_passes') else '?'}: loss {loss:.6f} vs {lo:.6f} ({le:.2e}) "
                      + " ".join(f"{n} {e:.1e}" for n, e in errs.items()), flush=True)
print("bad passes", bad, "of", iters * 9)
