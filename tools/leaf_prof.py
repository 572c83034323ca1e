"""Per-CTA phase stamps of the leaf GEMM (measurement only): entry, issue+clear done, first K group
landed, last K group landed, last FMA, exit — relative to the earliest entry, over a few steps.
    python tools/leaf_prof.py"""
import ctypes
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import synth
    from paper_conf_micro_khorasanieas18_b200 import vpps
    lib = ctypes.CDLL(os.path.join(ROOT, "paper_conf_micro_khorasanieas18_b200", "libvpps.so"))
    cfg = synth.CONFIGS["tgt"]
    H, E, C, V = cfg["H"], cfg["E"], cfg["C"], cfg["V"]
    rng = np.random.default_rng(0)
    shapes = vpps.param_shapes("binary", H, E, C)
    P = synth.init_params(shapes, rng)
    m = vpps.Model("binary", H, E, C, cluster=16, dataflow=True)
    params = torch.zeros(m.n_floats, device="cuda")
    grads = torch.zeros_like(params)
    for n, _ in shapes:
        m.views(params)[n].copy_(torch.from_numpy(P[n]).float())
    m.bind(params, grads)
    X = torch.from_numpy(synth.input_table(rng, V, E)).float().cuda()
    dX = torch.zeros_like(X)
    scripts = [m.build_script(synth.config_batch("tgt", i)) for i in range(4)]
    flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda")
    for i in range(5):
        m.fwd_bwd_sgd(scripts[i % 4], X, dX, lr=1e-3, weight_decay=0.0)
    torch.cuda.synchronize()
    buf = np.zeros(1024 * 8, dtype=np.uint64)
    for step in range(3):
        flush.zero_()
        lib.vpps_leaf_prof(1, None)
        torch.cuda.synchronize()
        m.fwd_bwd_sgd(scripts[step % 4], X, dX, lr=1e-3, weight_decay=0.0)
        torch.cuda.synchronize()
        lib.vpps_leaf_prof(0, None)
        lib.vpps_leaf_prof(0, buf.ctypes.data_as(ctypes.c_void_p))
        b = buf.reshape(1024, 8)[:148].astype(np.int64)
        t0 = b[:, 0].min()
        work = b[:, 2] > 0
        rel = (b - t0) / 1e3
        print(f"step {step}: CTAs {len(b)}, working {work.sum()}")
        names = ["entry", "issued / setup", "K0 landed", "K last landed", "FMA done", "exit", "clear done"]
        for k, nm in enumerate(names):
            sel = rel[work, k] if 2 <= k <= 5 else rel[:, k]
            print(f"  {nm:15s} min {sel.min():6.2f} mean {sel.mean():6.2f} max {sel.max():6.2f} us")
        b[:] = 0
        buf[:] = 0


if __name__ == "__main__":
    main()
