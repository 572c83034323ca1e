"""Throughput of the VPPS training step on every BASELINE.json config the GPU path covers (measurement only;
the graded bench line is bench.py's target config).

    python tools/config_sweep.py [--steps 50] [--warmup 5] [--out FILE]

Per case: 16 distinct pre-built, device-resident scripts cycled (each run once untimed first), fused forward + backward + SGD
(vpps_fwd_bwd_sgd), device time per step from CUDA events around the timed steps (no L2 flush: these are
steady-state numbers), samples/s, nodes/s and the algorithmic FLOP rate (SURVEY §8(d) F counted by the host
from the script) against the FP32 FFMA peak.
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

# (label, config, cell, H, E, C, V, batch, model options, overrides)
CASES = [
    ("c1 LSTM H32 B4", "c1", "lstm", 32, 32, 16, 16, 4, {}, {}),
    ("c1 LSTM H32 B4 (grid)", "c1", "lstm", 32, 32, 16, 16, 4, {"level": -1}, {}),
    ("c2 child-sum H128 B16", "c2", "childsum", 128, 128, 5, 4096, 16, {}, {}),
    ("c3 LSTM-LM H256 B1 (V=C=32)", "c3", "lstm", 256, 256, 32, 32, 1, {}, {"V": 32, "C": 32}),
    ("c3 LSTM-LM H256 B4 (V=C=32)", "c3", "lstm", 256, 256, 32, 32, 4, {}, {"V": 32, "C": 32}),
    ("c3 LSTM-LM H256 B16 (V=C=32)", "c3", "lstm", 256, 256, 32, 32, 16, {}, {"V": 32, "C": 32}),
    ("c3 LSTM-LM H256 B16 (V=C=32, grid)", "c3", "lstm", 256, 256, 32, 32, 16, {"level": -1}, {"V": 32, "C": 32}),
    ("c3 LSTM-LM H256 B64 (V=C=32)", "c3", "lstm", 256, 256, 32, 32, 64, {}, {"V": 32, "C": 32}),
    ("c2 child-sum H128 B16 G4", "c2", "childsum", 128, 128, 5, 4096, 16, {"groups": 4}, {}),
    ("c3 LSTM-LM H256 B16 G2", "c3", "lstm", 256, 256, 32, 32, 16, {"groups": 2}, {"V": 32, "C": 32}),
    ("c3 LSTM-LM H256 B64 G2", "c3", "lstm", 256, 256, 32, 32, 64, {"groups": 2}, {"V": 32, "C": 32}),
    ("c3 LSTM-LM H256 V1000 B1 (level path)", "c3", "lstm", 256, 256, 1000, 1000, 1, {}, {}),
    ("c3 LSTM-LM H256 V1000 B4 (level path)", "c3", "lstm", 256, 256, 1000, 1000, 4, {}, {}),
    ("c3 LSTM-LM H256 V1000 B16 (level path)", "c3", "lstm", 256, 256, 1000, 1000, 16, {}, {}),
    ("c3 LSTM-LM H256 V1000 B64 (level path)", "c3", "lstm", 256, 256, 1000, 1000, 64, {}, {}),
    ("GRU-LM H256 V1000 B4 (level path)", "c3", "gru", 256, 256, 1000, 1000, 4, {}, {}),
    ("GRU-LM H256 V1000 B16 (level path)", "c3", "gru", 256, 256, 1000, 1000, 16, {}, {}),
    ("GRU-LM H256 V1000 B64 (level path)", "c3", "gru", 256, 256, 1000, 1000, 64, {}, {}),
    ("RvNN H512 B16 (level path)", "tgt", "rvnn", 512, 512, 5, 4096, 16, {}, {}),
    ("RvNN H512 B64 (level path)", "tgt", "rvnn", 512, 512, 5, 4096, 64, {}, {}),
    ("TD-RNN H512 B16 (level path)", "tdrnn", "tdrnn", 512, 512, 5, 4096, 16, {}, {}),
    ("TD-LSTM H256 B16 (level path)", "tdrnn", "tdlstm", 256, 256, 5, 4096, 16, {}, {}),
    ("c4 BiLSTM tagger H512 B16 (level path)", "c4", "bilstm", 512, 512, 9, 4096, 16, {"mlp": 256}, {}),
    ("c5 binary H1024 B64 (level path)", "c5", "binary", 1024, 1024, 5, 4096, 64, {}, {}),
    ("BiLSTMwChar H256 E256 MLP256 B16 (chain)", "bilstmchar", "bilstmchar", 256, 256, 9, 4096, 16, {"mlp": 256}, {}),
    ("c4 BiLSTM tagger H512 B16 (per-step products)", "c4", "bilstm", 512, 512, 9, 4096, 16, {"mlp": 256, "chain": -1}, {}),
    ("tgt binary H256 B16 (level path)", "tgt", "binary", 256, 256, 5, 4096, 16, {"level": 1}, {}),
    ("tgt binary H128 E128 B16 (dataflow, 8-CTA groups)", "tgt", "binary", 128, 128, 5, 4096, 16, {"cluster": 8, "dataflow": True}, {}),
    ("tgt binary H128 E128 B16 (level path)", "tgt", "binary", 128, 128, 5, 4096, 16, {"level": 1}, {}),
    ("tgt binary H128 E128 B16 (grid)", "tgt", "binary", 128, 128, 5, 4096, 16, {"level": -1}, {}),
    ("c2 child-sum H128 B16 (auto groups)", "c2", "childsum", 128, 128, 5, 4096, 16, {"groups": -1}, {}),
    ("tgt binary H256 B16 (grid, auto groups)", "tgt", "binary", 256, 256, 5, 4096, 16, {"groups": -1, "level": -1}, {}),
    ("grid-G c1 LSTM H32 B4 G2", "c1", "lstm", 32, 32, 16, 16, 4, {"groups": 2, "level": -1}, {}),
    ("grid-G c1 LSTM H32 B4 G4", "c1", "lstm", 32, 32, 16, 16, 4, {"groups": 4, "level": -1}, {}),
    ("grid-G c2 child-sum H128 B16 G2", "c2", "childsum", 128, 128, 5, 4096, 16, {"groups": 2}, {}),
    ("grid-G tgt binary H256 B16 G1", "tgt", "binary", 256, 256, 5, 4096, 16, {"groups": 1, "level": -1}, {}),
    ("grid-G tgt binary H256 B16 G2", "tgt", "binary", 256, 256, 5, 4096, 16, {"groups": 2, "level": -1}, {}),
    ("grid-G tgt binary H256 B16 G4", "tgt", "binary", 256, 256, 5, 4096, 16, {"groups": 4, "level": -1}, {}),
    ("grid-G tgt binary H128 B16 G4", "tgt", "binary", 128, 128, 5, 4096, 16, {"groups": 4, "level": -1}, {}),
    ("grid-G c3 LSTM-LM H256 B16 (V=C=32) G4", "c3", "lstm", 256, 256, 32, 32, 16, {"groups": 4, "level": -1}, {"V": 32, "C": 32}),
    ("tgt binary H256 B1 (dataflow)", "tgt", "binary", 256, 256, 5, 4096, 1, {"cluster": 16, "dataflow": True}, {}),
    ("tgt binary H256 B4 (dataflow)", "tgt", "binary", 256, 256, 5, 4096, 4, {"cluster": 16, "dataflow": True}, {}),
    ("tgt binary H256 B16 (dataflow)", "tgt", "binary", 256, 256, 5, 4096, 16, {"cluster": 16, "dataflow": True}, {}),
    ("tgt binary H256 B64 (dataflow)", "tgt", "binary", 256, 256, 5, 4096, 64, {"cluster": 16, "dataflow": True}, {}),
]


def kernel_label(cell, H, C, opts):
    if opts.get("dataflow"):
        return "vpps_df + GEMMs"
    lvl = opts.get("level", 0)
    if cell in ("lstm", "childsum", "binary") and lvl == -1:
        return "vpps_fb (grid)"
    chain = cell in ("bilstm", "gru", "bilstmchar") or (
        cell == "lstm" and opts.get("groups", 1) <= 1 and (lvl > 0 or C > 32 or H >= 128))
    if chain and os.environ.get("VPPS_CHAIN", "1") != "0" and opts.get("chain", 0) >= 0 and H in (32, 64, 128, 256, 512):
        return "vpps_chain (register-resident recurrence) + GEMMs"
    if opts.get("level") or H > 256 or cell in ("bilstm", "gru", "rvnn", "tdrnn", "tdlstm") or C > 32:
        return "level GEMMs"
    return "vpps_fb (grid)"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=16,
                    help="untimed passes; >= 16 runs every script once, so work buffers that grow with the "
                         "largest script are allocated before the timed region")
    ap.add_argument("--out", default=None)
    ap.add_argument("--only", default=None, help="run the cases whose label contains this substring")
    args = ap.parse_args()
    import torch
    import synth
    from paper_conf_micro_khorasanieas18_b200 import vpps
    mhz = 1965.0
    peak = 148 * 128 * 2 * mhz * 1e6
    lines = []
    for label, cfg, cell, H, E, C, V, B, opts, over in CASES:
        if args.only and args.only not in label:
            continue
        rng = np.random.default_rng(0)
        shapes = vpps.param_shapes(cell, H, E, C, opts.get("mlp", 256))
        P = synth.init_params(shapes, rng)
        try:
            m = vpps.Model(cell, H, E, C, **opts)
        except Exception as e:   # noqa: BLE001 (a config the GPU path does not cover)
            lines.append({"case": label, "error": str(e)})
            print(json.dumps(lines[-1]), flush=True)
            continue
        params = torch.zeros(m.n_floats, device="cuda")
        grads = torch.zeros_like(params)
        for n, _ in shapes:
            m.views(params)[n].copy_(torch.from_numpy(P[n]).float())
        m.bind(params, grads)
        X = torch.from_numpy(synth.input_table(rng, V, E)).float().cuda()
        dX = torch.zeros_like(X)
        scripts, flops, nodes = [], [], []
        for b in range(16):
            g = synth.config_batch(cfg, b, batch=B, **over)
            s = m.build_script(g)
            s.upload()
            scripts.append(s)
            inf = s.info()
            flops.append(inf["flops"])
            nodes.append(inf["n_nodes"])
        for i in range(args.warmup):
            m.fwd_bwd_sgd(scripts[i % 16], X, dX, lr=1e-4)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for i in range(args.steps):
            m.fwd_bwd_sgd(scripts[i % 16], X, dX, lr=1e-4)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / args.steps
        f = float(np.mean([flops[i % 16] for i in range(args.steps)]))
        nn = float(np.mean([nodes[i % 16] for i in range(args.steps)]))
        rec = {"case": label, "ms_per_step": round(ms, 4), "samples_per_s": round(B / ms * 1e3, 1),
               "nodes_per_s": round(nn / ms * 1e3, 1), "gflop_per_step": round(f / 1e9, 4),
               "tflops": round(f / ms / 1e9, 3), "frac_fp32_peak": round(f / (ms * 1e-3) / peak, 4),
               "kernel": kernel_label(cell, H, C, opts)}
        lines.append(rec)
        print(json.dumps(rec), flush=True)
        del m
    if args.out:
        with open(args.out, "w") as fh:
            for r in lines:
                fh.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
