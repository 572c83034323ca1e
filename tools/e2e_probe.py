"""Where the end-to-end step goes: host enqueue time per call, e2e loop with 1-4 prefetch workers,
with and without the per-step stale-loss read (TGT, no L2 flush)."""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    import synth
    from paper_conf_micro_khorasanieas18_b200 import vpps
    H = E = 256
    C = 5
    rng = np.random.default_rng(0)
    shapes = vpps.param_shapes("binary", H, E, C)
    P = synth.init_params(shapes, rng)
    m = vpps.Model("binary", H, E, C, cluster=16, dataflow=True)
    params = torch.zeros(m.n_floats, device="cuda")
    grads = torch.zeros_like(params)
    for n, _ in shapes:
        m.views(params)[n].copy_(torch.from_numpy(P[n]).float())
    m.bind(params, grads)
    X = torch.from_numpy(synth.input_table(rng, 4096, E)).float().cuda()
    dX = torch.zeros_like(X)
    csr = [vpps.CsrBatch.from_graphs(synth.config_batch("tgt", i)) for i in range(64)]
    scripts = [m.build_script(c) for c in csr]
    for i in range(30):
        m.fwd_bwd_sgd(scripts[i % 64], X, dX, lr=1e-3)
    torch.cuda.synchronize()
    # host enqueue cost of one call (device far behind: measure the call itself)
    t = time.perf_counter()
    for i in range(200):
        m.fwd_bwd_sgd(scripts[i % 64], X, dX, lr=1e-3)
    th = (time.perf_counter() - t) / 200
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for i in range(200):
        m.fwd_bwd_sgd(scripts[i % 64], X, dX, lr=1e-3)
    e1.record()
    torch.cuda.synchronize()
    print(f"host enqueue {th * 1e6:.1f} us/call; device back-to-back {e0.elapsed_time(e1) / 200 * 1e3:.1f} us/step")
    for w in (1, 2, 3, 4):
        for stale in (True, False):
            torch.cuda.synchronize()
            t = time.perf_counter()
            n = 300
            for k, s in enumerate(vpps.prefetch_scripts(m, (csr[k % 64] for k in range(n)), workers=w)):
                m.fwd_bwd_sgd(s, X, dX, lr=1e-3)
                if stale and k > 0:
                    m.stale_loss()
            m.latest_loss()
            dt = (time.perf_counter() - t) / n
            print(f"e2e workers {w} stale-loss {stale}: {dt * 1e6:.1f} us/step = {16 / dt / 1e3:.1f} K samples/s")


if __name__ == "__main__":
    main()
