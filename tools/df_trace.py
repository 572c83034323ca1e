"""Section clocks of the dataflow kernel (vpps_df) from its in-kernel trace (vpps_set_profile_buffer).

    python tools/df_trace.py [--batch-idx 0] [--reps 3]

Per CTA: span (globaltimer), batches executed and cycles per section (0 program decode, 1 staging issue,
2 tag wait / data arrival, 3 forward, 4 cell-bwd, 5 transposed product, 6 heads, 7 other).  Prints the
mean over CTAs, the slowest CTA and the per-group spans.
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
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--config", default="tgt")
    ap.add_argument("--batches", action="store_true", help="per-batch timeline of the last CTA's group")
    ap.add_argument("--sgd", action="store_true", help="fused SGD step (the bench mode)")
    ap.add_argument("--flush", action="store_true", help="256 MiB L2 flush before the traced pass (the bench mode)")
    args = ap.parse_args()
    import torch
    import synth
    from paper_conf_micro_khorasanieas18_b200 import vpps
    cfg = synth.CONFIGS[args.config]
    cell, H, E, C, V = cfg["cell"], cfg["H"], cfg["E"], cfg["C"], cfg["V"]
    rng = np.random.default_rng(0)
    shapes = vpps.param_shapes(cell, H, E, C)
    P = synth.init_params(shapes, rng)
    m = vpps.Model(cell, H, E, C, cluster=16, dataflow=True)
    params = torch.zeros(m.n_floats, device="cuda")
    grads = torch.zeros_like(params)
    for n, _ in shapes:
        m.views(params)[n].copy_(torch.from_numpy(P[n]).float())
    m.bind(params, grads)
    X = torch.from_numpy(synth.input_table(rng, V, E)).float().cuda()
    dX = torch.zeros_like(X)
    s = m.build_script(synth.config_batch(args.config, args.batch_idx))
    n_cta = m.plan_info()["n_cta"]
    stride = 16 + 5 * 48 + 32
    buf = torch.zeros((n_cta, stride), dtype=torch.int64, device="cuda")
    m.set_profile_buffer(buf, stride)
    gt = torch.zeros((4096, 5), dtype=torch.int64, device="cuda")
    m.set_gemm_trace(gt)
    for r in range(args.reps):
        if r == args.reps - 1:
            torch.cuda.synchronize()
            buf.zero_()
            if args.flush:
                torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda").zero_()
                torch.cuda.synchronize()
        if args.sgd:
            m.fwd_bwd_sgd(s, X, dX, lr=1e-3)
        else:
            m.fwd_bwd(s, X, dX)
    torch.cuda.synchronize()
    raw = buf.cpu().numpy().astype(np.float64)
    gtr = gt.cpu().numpy().astype(np.float64)
    tail = gtr[3000:][gtr[3000:, 0] == 99]
    gtr = gtr[:3000]
    gtr = gtr[gtr[:, 3] > 0]
    t0 = raw[:, 0].min()
    span = (raw[:, 1] - raw[:, 0]) / 1e3
    if raw[:, 11].min() > 0:
        print(f"kernel entry skew {(raw[:, 11].max() - raw[:, 11].min()) / 1e3:.1f} us, prologue (entry -> span "
              f"start) mean {((raw[:, 0] - raw[:, 11]) / 1e3).mean():.1f} max {((raw[:, 0] - raw[:, 11]) / 1e3).max():.1f} us, "
              f"epilogue (span end -> exit) mean {((raw[:, 12] - raw[:, 1]) / 1e3).mean():.1f} max "
              f"{((raw[:, 12] - raw[:, 1]) / 1e3).max():.1f} us, first entry -> last exit "
              f"{(raw[:, 12].max() - raw[:, 11].min()) / 1e3:.1f} us")
    names = ["program", "staging", "tag-wait", "forward", "cell-bwd", "transp", "heads", "other"]
    secs = raw[:, 3:11]
    print(f"{args.config} batch {args.batch_idx}: {n_cta} CTAs, span max {span.max():.1f} us "
          f"(start skew {(raw[:, 0].max() - t0) / 1e3:.1f} us)")
    groups = n_cta // 16
    print("group spans (us): " + ", ".join(f"{(raw[g*16:(g+1)*16, 1].max() - t0) / 1e3:.1f}" for g in range(groups)))
    print("batches per group: " + ", ".join(f"{int(raw[g*16, 2])}" for g in range(groups)))
    if len(gtr):
        gend = [(raw[g*16:(g+1)*16, 1].max() - t0) / 1e3 for g in range(groups)]
        st = (gtr[:, 2] - t0) / 1e3
        en = (gtr[:, 3] - t0) / 1e3
        if len(tail):
            ts, te = (tail[:, 2] - t0) / 1e3, (tail[:, 3] - t0) / 1e3
            print(f"gradient GEMM tail ({len(tail)} CTAs): fin seen {ts.min():.1f}-{ts.max():.1f} us, "
                  f"SGD + exit {te.min():.1f}-{te.max():.1f} us")
        print(f"gradient GEMM: {len(gtr)} items, first start {st.min():.1f} us, last end {en.max():.1f} us, "
              f"mean item {np.mean(en - st):.2f} us, SMs used {len(set(gtr[:, 4]))}")
        for g in range(groups):
            sel = gtr[:, 0] == g
            if sel.any():
                print(f"  group {g}: done {gend[g]:.1f} us; its {int(sel.sum())} items run {st[sel].min():.1f}-{en[sel].max():.1f} us")
        kern_end = (raw[:, 1].max() - t0) / 1e3
        print(f"  items finished before the last group ended: {(en <= kern_end).mean()*100:.0f} %")
        # the last group's items: how they spread over SMs (items sharing an SM run slower)
        gl = int(np.argmax(gend))
        sel = gtr[:, 0] == gl
        sms = gtr[sel, 4].astype(int)
        cnt = np.bincount(sms, minlength=160)
        dur = en[sel] - st[sel]
        occ = []
        for k in np.nonzero(sel)[0]:
            same = (gtr[:, 4] == gtr[k, 4]) & (st < en[k]) & (en > st[k])
            occ.append(int(same.sum()))
        occ = np.array(occ)
        print(f"  last group {gl}: {int(sel.sum())} items on {int((cnt > 0).sum())} SMs (max {int(cnt.max())} per SM); "
              f"item time {dur.min():.1f}-{dur.max():.1f} us; items overlapping on their SM: "
              + ", ".join(f"{v}: {int((occ == v).sum())}" for v in sorted(set(occ.tolist()))))
    mean = secs.mean(0)
    slow = secs[np.argmax(raw[:, 1])]
    tot = mean.sum()
    print("section kcycles (mean | CTA that finished last):")
    print("  " + ", ".join(f"{n} {a/1e3:.0f}k ({a/tot*100:.0f}%) | {b/1e3:.0f}k" for n, a, b in zip(names, mean, slow)))
    if args.batches:
        last = int(np.argmax(raw[:, 1]))
        g0 = (last // 16) * 16
        ops = {0x20: "LEAF_F", 0x21: "LEAF_B", 0x22: "INT_F", 0x23: "INT_B", 0x42: "HEAD_FB"}
        print(f"per-batch cycles of group {last // 16} (CTA {g0} | CTA {last}): issue->staged, staged->fresh "
              f"(retry rounds), compute, batch end relative to CTA {g0}")
        nbt = int(raw[last, 2])
        for cta in (g0,):
            b = raw[cta, 16:16 + 5 * 48].reshape(48, 5)
            bl = raw[last, 16:16 + 5 * 48].reshape(48, 5)
            for k in range(min(nbt, 48)):
                op = int(b[k, 4]) & 0xFF
                r = int(b[k, 4]) >> 8
                print(f"  {k:3d} {ops.get(op, hex(op)):7s} stage {b[k,1]-b[k,0]:6.0f} wait {b[k,2]-b[k,1]:6.0f} ({r} rnd)"
                      f" compute {b[k,3]-b[k,2]:6.0f} | end skew vs last CTA {bl[k,3]-b[k,3]:7.0f}")
            x = raw[cta, 256:288]
            if x[0] > 0:
                print("  INT_F nb=1 compute: fma %.0f, reduce %.0f, cell+stores %.0f, end barrier %.0f" %
                      (x[1] - x[0], x[2] - x[1], x[3] - x[2], x[4] - x[3]))
            if x[16] > 0:
                print("  INT_F nb=1 staging: issue %.0f, cp.async wait %.0f, bar %.0f, check %.0f, bar_count %.0f" %
                      (x[17] - x[16], x[18] - x[17], x[19] - x[18], x[20] - x[19], x[0] - x[20]))
            if x[22] > 0:
                print("  INT_B nb=1 staging: issue %.0f, cp.async wait %.0f, poll %.0f, bar %.0f" %
                      (x[23] - x[22], x[24] - x[23], x[25] - x[24], x[26] - x[25]))
            if x[5] > 0:
                print("  INT_B nb=1 compute: cell-bwd %.0f, tmv+sts %.0f, bar %.0f, reduce+st %.0f, bar %.0f, end bar %.0f" %
                      (x[6] - x[5], x[7] - x[6], x[8] - x[7], x[9] - x[8], x[10] - x[9], x[11] - x[10]))
            if x[27] > 0:
                print("  INT_B big batch: staging %.0f, cell-bwd %.0f, transposed chunks %.0f, end bar %.0f" %
                      (x[28] - x[27], x[29] - x[28], x[30] - x[29], x[31] - x[30]))
            if x[12] > 0:
                print("  LEAF_B iter0: poll %.0f, compute+stores %.0f; loop total from iter0 issue %.0f" %
                      (x[13] - x[12], x[14] - x[13], x[15] - x[12]))


if __name__ == "__main__":
    main()
