"""Per-phase timeline of one VPPS pass from the in-kernel %globaltimer trace (vpps_set_profile_buffer).

    python tools/phase_trace.py [--batch-idx 0] [--reps 5]

Phase p = forward level p (p <= L) or backward level 2L+1-p.  For each phase: the slowest CTA's work time
(wait-end of barrier p -> signal of barrier p+1), the mean over CTAs, and the barrier latency (last signal
of barrier p -> first/last release).  Prints a summary of barrier vs work share.
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch-idx", type=int, default=0)
    ap.add_argument("--reps", type=int, default=1)
    ap.add_argument("--config", default="tgt")
    ap.add_argument("--groups", type=int, default=1)
    ap.add_argument("--quiet", action="store_true")
    ap.add_argument("--sections", action="store_true")
    ap.add_argument("--cluster", type=int, default=0)
    ap.add_argument("--vocab", type=int, default=0, help="override V = C (e.g. 32 for the config-3 GPU reading)")
    ap.add_argument("--batch", type=int, default=0)
    args = ap.parse_args()
    import torch
    import synth
    from paper_conf_micro_khorasanieas18_b200 import vpps
    cfg = synth.CONFIGS[args.config]
    cell, H, E, C, V = cfg["cell"], cfg["H"], cfg["E"], cfg["C"], cfg["V"]
    over = {}
    if args.vocab:
        C = V = args.vocab
        over = {"V": V, "C": C}
    rng = np.random.default_rng(0)
    shapes = vpps.param_shapes(cell, H, E, C)
    P = synth.init_params(shapes, rng)
    m = vpps.Model(cell, H, E, C, groups=args.groups, cluster=args.cluster)
    params = torch.zeros(m.n_floats, device="cuda")
    grads = torch.zeros_like(params)
    for n, _ in shapes:
        m.views(params)[n].copy_(torch.from_numpy(P[n]).float())
    m.bind(params, grads)
    X = torch.from_numpy(synth.input_table(rng, V, E)).float().cuda()
    dX = torch.zeros_like(X)
    graphs = synth.config_batch(args.config, args.batch_idx, batch=args.batch or None, **over)
    s = m.build_script(graphs)
    info = s.info()
    nbar = info["n_barriers"]
    n_cta = m.plan_info()["n_cta"]
    n_act = m.plan_info()["n_act"]
    stride = 2 + 3 * (nbar + 1) + 10 * (nbar + 2)
    buf = torch.zeros((n_cta, stride), dtype=torch.int64, device="cuda")
    m.set_profile_buffer(buf, stride)
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
    for _ in range(args.reps):
        ev[0].record()
        m.fwd_bwd(s, X, dX)
        ev[1].record()
    torch.cuda.synchronize()
    kernel_us = ev[0].elapsed_time(ev[1]) * 1e3
    n_g = m.plan_info()["n_g"]
    raw = buf.cpu().numpy().astype(np.float64)
    rows = [c for c in range(n_cta) if c % n_g < n_act]
    t = raw[rows]
    t[t == 0] = np.nan                       # stamps of phases a group did not take part in
    t0 = np.nanmin(t[:, 0])
    t = t - t0
    L = (nbar - 1) // 2
    # node counts per phase from the script words (cell/head instructions of stream 0)
    from oracle import script as osc   # test infrastructure: only to label phases with node counts
    ref = osc.build(cell, graphs, H, E, C, 1, n_act)
    lv = ref["levels"]
    counts = [sum(1 for x in lv if x == (p if p <= L else 2 * L + 1 - p)) for p in range(nbar + 1)]
    print(f"{args.config}: {len(graphs)} graphs, {info['n_nodes']} nodes, {nbar} barriers, kernel "
          f"{kernel_us:.1f} us (event, incl. memsets), trace span {np.nanmax(t[:, 1]):.0f} ns, groups {args.groups}")
    work_tot = bar_tot = 0.0
    if not args.quiet:
        print(" phase  nodes   work_max   work_mean   barrier(last sig->last release)")
    for p in range(nbar + 1):
        start = t[:, 0] if p == 0 else t[:, 4 + 3 * p]
        end = t[:, 1] if p == nbar else t[:, 2 + 3 * (p + 1)]
        w = end - start
        bl = 0.0
        if p >= 1:
            bl = np.nanmax(t[:, 2 + 3 * p + 2]) - np.nanmax(t[:, 2 + 3 * p])
        wmax = np.nanmax(w) if np.any(~np.isnan(w)) else 0.0
        wmean = np.nanmean(w) if np.any(~np.isnan(w)) else 0.0
        work_tot += wmax
        bar_tot += bl
        if not args.quiet:
            print(f" {p:5d} {counts[p]:6d} {wmax/1e3:9.2f}us {wmean/1e3:9.2f}us {bl/1e3:9.2f}us")
    print(f"sum work_max {work_tot/1e3:.1f} us, sum barrier {bar_tot/1e3:.1f} us")
    secs = raw[rows][:, 2 + 3 * (nbar + 1): 2 + 3 * (nbar + 1) + 10]
    names = ["decode", "staging", "matvec", "cell", "cell-bwd", "outer/tmv", "heads", "signal", "wait", "other"]
    if args.cluster:
        names = ["decode", "staging", "forward", "cell-bwd", "transp", "heads", "arrive", "wait", "tail", "other"]
    mean = secs.mean(0)
    mx = secs[secs.sum(1).argmax()]
    tot = mean.sum()
    print("section cycles (mean over CTAs | slowest CTA):")
    print("  " + ", ".join(f"{n} {m/1e3:.0f}k ({m/tot*100:.0f}%) | {x/1e3:.0f}k" for n, m, x in zip(names, mean, mx)))
    if args.sections:
        # per-phase section clocks of CTA 0 (cumulative snapshots at each signal)
        base = 2 + 3 * (nbar + 1) + 10
        cum = raw[0, base: base + 10 * (nbar + 1)].reshape(nbar + 1, 10)
        final = raw[0, 2 + 3 * (nbar + 1): 2 + 3 * (nbar + 1) + 10]
        cum = np.vstack([cum[1:], final])            # snapshot b = end of phase b-1
        prev = np.zeros(10)
        print(" phase " + " ".join(f"{n[:8]:>8s}" for n in names) + "   (kcycles, CTA 0)")
        for p in range(nbar + 1):
            d = cum[p] - prev
            prev = cum[p]
            print(f" {p:5d} " + " ".join(f"{v/1e3:8.1f}" for v in d))


if __name__ == "__main__":
    main()
