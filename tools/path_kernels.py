"""Per-kernel device time of one training step on any device path (measurement only): the CUDA activity
trace of torch.profiler (CUPTI kernel records) over a few steady-state steps, kernels grouped by name,
with their share of the summed kernel time and the launch count per step.

    python tools/path_kernels.py --case c5 [--steps 5]
cases: c5 (binary H1024 B64, level path), c4 (BiLSTM tagger H512 B16, chain), c3 (LSTM LM H256 V1000 B64,
chain), tgt (binary H256 B16, dataflow)
"""
import argparse
import collections
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

CASES = {
    "c5": ("c5", "binary", 1024, 1024, 5, 4096, 64, {}, {}),
    "c4": ("c4", "bilstm", 512, 512, 9, 4096, 16, {"mlp": 256}, {}),
    "c3": ("c3", "lstm", 256, 256, 1000, 1000, 64, {}, {}),
    "tgt": ("tgt", "binary", 256, 256, 5, 4096, 16, {"cluster": 16, "dataflow": True}, {}),
}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--case", default="c5", choices=sorted(CASES))
    ap.add_argument("--steps", type=int, default=5)
    args = ap.parse_args()
    import torch
    import synth
    from paper_conf_micro_khorasanieas18_b200 import vpps
    cfg, cell, H, E, C, V, B, opts, over = CASES[args.case]
    rng = np.random.default_rng(0)
    shapes = vpps.param_shapes(cell, H, E, C, opts.get("mlp", 256))
    P = synth.init_params(shapes, rng)
    m = vpps.Model(cell, H, E, C, **opts)
    params = torch.zeros(m.n_floats, device="cuda")
    grads = torch.zeros_like(params)
    for n, _ in shapes:
        m.views(params)[n].copy_(torch.from_numpy(P[n]).float())
    m.bind(params, grads)
    X = torch.from_numpy(synth.input_table(rng, V, E)).float().cuda()
    dX = torch.zeros_like(X)
    scripts = [m.build_script(synth.config_batch(cfg, i, batch=B, **over)) for i in range(4)]
    for s in scripts:
        s.upload()
    for i in range(8):
        m.fwd_bwd_sgd(scripts[i % 4], X, dX, lr=1e-4)
    torch.cuda.synchronize()
    from torch.profiler import ProfilerActivity, profile
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        e0.record()
        for i in range(args.steps):
            m.fwd_bwd_sgd(scripts[i % 4], X, dX, lr=1e-4)
        e1.record()
        torch.cuda.synchronize()
    wall = e0.elapsed_time(e1) / args.steps
    agg = collections.defaultdict(lambda: [0, 0.0])
    for ev in prof.events():
        if ev.device_type.name != "CUDA" or ev.device_time_total <= 0:
            continue
        name = ev.name.split("(")[0][:70]
        agg[name][0] += 1
        agg[name][1] += ev.device_time_total
    tot = sum(v[1] for v in agg.values())
    print(f"case {args.case}: {wall:.3f} ms per step (events, profiler attached); kernel time {tot / args.steps / 1e3:.3f} ms per step")
    print(f"{'kernel':72s} {'launches/step':>13s} {'ms/step':>8s} {'share':>6s}")
    for name, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1])[:25]:
        print(f"{name:72s} {n / args.steps:13.1f} {t / args.steps / 1e3:8.3f} {t / tot * 100:5.1f}%")


if __name__ == "__main__":
    main()
