"""Per-kernel device times of one VPPS training step under bench conditions (warm launch queue, L2 flushed
before each step, intermediate data L2-resident as in a real step) via the CUDA activity trace of
torch.profiler (CUPTI kernel records; no replay, no serialisation).

    python tools/kernel_times.py [--steps 20] [--cluster 16] [--groups 4] [--no-flush]
"""
import argparse
import collections
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--cluster", type=int, default=16)
    ap.add_argument("--groups", type=int, default=4)
    ap.add_argument("--config", default="tgt")
    ap.add_argument("--no-flush", action="store_true")
    ap.add_argument("--sync", choices=["dataflow", "cluster"], default="dataflow")
    args = ap.parse_args()
    import torch
    import synth
    from paper_conf_micro_khorasanieas18_b200 import vpps
    cfg = synth.CONFIGS[args.config]
    cell, H, E, C, V = cfg["cell"], cfg["H"], cfg["E"], cfg["C"], cfg["V"]
    rng = np.random.default_rng(0)
    shapes = vpps.param_shapes(cell, H, E, C)
    P = synth.init_params(shapes, rng)
    m = vpps.Model(cell, H, E, C, groups=args.groups, cluster=args.cluster, dataflow=args.sync == "dataflow")
    params = torch.zeros(m.n_floats, device="cuda")
    grads = torch.zeros_like(params)
    for n, _ in shapes:
        m.views(params)[n].copy_(torch.from_numpy(P[n]).float())
    m.bind(params, grads)
    X = torch.from_numpy(synth.input_table(rng, V, E)).float().cuda()
    dX = torch.zeros_like(X)
    scripts = [m.build_script(synth.config_batch(args.config, i)) for i in range(16)]
    for s in scripts:
        s.upload()
    flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda")
    for i in range(5):
        m.fwd_bwd_sgd(scripts[i % 16], X, dX, lr=1e-3, weight_decay=0.0)
    torch.cuda.synchronize()
    from torch.profiler import ProfilerActivity, profile
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for i in range(args.steps):
            if not args.no_flush:
                flush.zero_()
            m.fwd_bwd_sgd(scripts[i % 16], X, dX, lr=1e-3, weight_decay=0.0)
        torch.cuda.synchronize()
    # timeline of the last few steps: kernel start / end relative to the step's first kernel (us)
    evs = sorted([e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA],
                 key=lambda e: e.time_range.start)
    steps, cur = [], []
    for e in evs:
        if "leaf_fwd" in e.name and cur:
            steps.append(cur)
            cur = []
        if "FillFunc" not in e.name:
            cur.append(e)
    if cur:
        steps.append(cur)
    for st in steps[-3:]:
        t0 = st[0].time_range.start
        print("step timeline (us): " + "; ".join(
            f"{e.name.split('(')[0].split('::')[-1][:18]} {e.time_range.start - t0:.1f}-{e.time_range.end - t0:.1f}"
            for e in st))
    per = collections.defaultdict(list)
    for e in prof.events():
        if e.device_type == torch.autograd.DeviceType.CUDA:
            per[e.name[:70]].append(e.device_time_total if hasattr(e, "device_time_total") else e.cuda_time_total)
    tot = 0.0
    print(f"{'kernel':70s} {'n':>4s} {'mean us':>9s}")
    for k, v in sorted(per.items(), key=lambda kv: -sum(kv[1])):
        if "FillFunc" in k and not args.no_flush and len(v) == args.steps:
            name = k + " (L2 flush, not in step)"
        else:
            name = k
            tot += sum(v) / args.steps
        print(f"{name[:70]:70s} {len(v):4d} {np.mean(v):9.1f}")
    print(f"sum of per-step device time (excluding the flush): {tot:.1f} us")


if __name__ == "__main__":
    main()
