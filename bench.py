#!/usr/bin/env python
"""VPPS benchmark: binary Tree-LSTM (H = E = 256) training samples/s on N B200s (BASELINE.json).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl vpps|reference] [--batch B]

One step = one pass of the whole hot path on one batch of B synthetic SST-shaped trees per GPU:
  N = 1: vpps_fwd_bwd_sgd — forward, backward and SGD update in one persistent kernel
  N > 1: vpps_fwd_bwd -> NCCL all-reduce of the flat gradient -> vpps_sgd_step (weak scaling)
64 distinct pre-built batches per rank are cycled (every step sees a new graph shape, L44); the L2 is
flushed (256 MiB write) before every timed step, outside the timed region.  Rank 0 prints one JSON line.
`--impl reference` times the FP64 CPU oracle (oracle/) on the same workload (bounded sample per step).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402

METRIC = "Tree-LSTM training samples/sec at 1/2/4/8 B200; DRAM bytes/pass vs weights-once"
H = E = 256
C = 5
V = 4096
N_BATCHES = 64
WORKLOAD = ("tgt: binary Tree-LSTM (M4) H=E=256, C=5, SST-shaped synthetic trees with 5-50 leaves, "
            "input table 4096x256, fwd+bwd+dX+SGD")


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def fp32_peak_tflops(mhz: float) -> float:
    """FP32 FFMA peak: 148 SMs x 128 FP32 lanes x 2 FLOP x SM clock."""
    return 148 * 128 * 2 * mhz * 1e6 / 1e12


class ClockSampler:
    """SM clocks and throttle reasons sampled during the timed region (B200_PROFILING.md): NVML polled
    every ~2 ms from a thread (the timed region can be tens of ms), nvidia-smi as the fallback."""

    REASONS = {"hw_slowdown": 0x8, "hw_thermal_slowdown": 0x40, "sw_thermal_slowdown": 0x20, "sw_power_cap": 0x4}

    def __init__(self, index: int):
        self.index = index
        self.sm, self.max_sm, self.mask = [], None, 0
        self.stop_ev = threading.Event()
        self.thread = None
        self.nvml = None

    def start(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self.max_sm = float(pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM))
            self.nvml = (pynvml, h)
        except Exception:
            self.nvml = None
        self.thread = threading.Thread(target=self._poll, daemon=True)
        self.thread.start()

    def _poll(self):
        if self.nvml:
            pynvml, h = self.nvml
            while not self.stop_ev.is_set():
                try:
                    self.sm.append(float(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)))
                    self.mask |= int(pynvml.nvmlDeviceGetCurrentClocksEventReasons(h))
                except Exception:
                    break
                time.sleep(0.002)
            return
        q = "clocks.sm,clocks.max.sm,clocks_event_reasons.active"
        while not self.stop_ev.is_set():
            try:
                out = subprocess.run(["nvidia-smi", f"--id={self.index}", f"--query-gpu={q}",
                                      "--format=csv,noheader,nounits"], capture_output=True, text=True,
                                     timeout=5).stdout.strip().split(",")
                self.sm.append(float(out[0]))
                self.max_sm = float(out[1])
                self.mask |= int(out[2], 16)
            except Exception:
                break

    def stop(self):
        self.stop_ev.set()
        if self.thread:
            self.thread.join(timeout=10)
        if not self.sm:
            return {"sm_mhz": None, "sm_max_mhz": self.max_sm, "reasons": ["unsampled"]}
        reasons = sorted(n for n, bit in self.REASONS.items() if self.mask & bit)
        return {"sm_mhz": statistics.median(self.sm), "sm_max_mhz": self.max_sm, "reasons": reasons,
                "samples": len(self.sm), "source": "nvml" if self.nvml else "nvidia-smi"}


PROFILE_TAG = "r2f"     # profiles/<tag>_ncu_summary.json: ncu capture of the kernels this bench times


def make_batches(rank: int, batch: int):
    # rank r's batches are config 'tgt' batches r*N_BATCHES .. r*N_BATCHES+63 (disjoint shards)
    return [synth.config_batch("tgt", rank * N_BATCHES + i, batch=batch) for i in range(N_BATCHES)]


def run_reference(args, world: int, rank: int):
    """--impl reference: the FP64 oracle as it stands, on the host cores, rank 0 only."""
    if rank != 0:
        return
    from threadpoolctl import threadpool_limits
    from oracle import models as M
    rng = np.random.default_rng(0)
    P = synth.init_params(M.param_shapes("binary", H, E, C), rng)
    X = synth.input_table(rng, V, E)
    batches = make_batches(0, args.batch)
    per_step = 1                     # bounded sample: one tree of the step's batch per step
    with threadpool_limits(limits=1):
        for w in range(args.warmup):
            M.forward_backward("binary", P, X, batches[w % N_BATCHES][:per_step], H)
        t0 = time.perf_counter()
        for k in range(args.steps):
            g = batches[k % N_BATCHES]
            M.forward_backward("binary", P, X, [g[k % len(g)]], H)
        dt = time.perf_counter() - t0
    value = args.steps * per_step / dt
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "samples/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * dt / args.steps,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": WORKLOAD, "global_batch": args.batch * world, "per_gpu_batch": args.batch,
                   "parallelism": f"dp{world}"},
        "cpu_baseline": {"value": value, "unit": "samples/s", "cores": 1, "kind": "oracle", "cpu": lscpu_model(),
                         "sample": f"{per_step} tree of each step's batch (FP64 NumPy, BLAS threads = 1)"},
        "e2e": {"value": value, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def cpu_baseline(batches, budget_s=12.0):
    """Oracle timed on a bounded sample of the same workload (1 thread)."""
    from threadpoolctl import threadpool_limits
    from oracle import models as M
    rng = np.random.default_rng(0)
    P = synth.init_params(M.param_shapes("binary", H, E, C), rng)
    X = synth.input_table(rng, V, E)
    n, t0 = 0, time.perf_counter()
    with threadpool_limits(limits=1):
        for g in batches:
            for tree in g:
                M.forward_backward("binary", P, X, [tree], H)
                n += 1
                if time.perf_counter() - t0 > budget_s:
                    break
            if time.perf_counter() - t0 > budget_s:
                break
    dt = time.perf_counter() - t0
    return {"value": n / dt, "unit": "samples/s", "cores": 1, "kind": "oracle", "cpu": lscpu_model(),
            "sample": f"{n} trees of the bench batches in {dt:.1f} s (FP64 NumPy, BLAS threads = 1)"}


def _oracle_trees(args_):
    """Worker of cpu_baseline_all_cores: trees (b, i) of the bench batches through the FP64 oracle."""
    idx, budget_s = args_
    from threadpoolctl import threadpool_limits
    from oracle import models as M
    rng = np.random.default_rng(0)
    P = synth.init_params(M.param_shapes("binary", H, E, C), rng)
    X = synth.input_table(rng, V, E)
    batches = make_batches(0, 16)
    n, t0 = 0, time.perf_counter()
    with threadpool_limits(limits=1):
        for b, i in idx:
            M.forward_backward("binary", P, X, [batches[b][i]], H)
            n += 1
            if time.perf_counter() - t0 > budget_s:
                break
    return n


def cpu_baseline_all_cores(batches, budget_s=8.0):
    """The same oracle across every host core (one process per core, trees split round-robin)."""
    import multiprocessing as mp
    cores = len(os.sched_getaffinity(0))
    trees = [(b, i) for b in range(len(batches)) for i in range(len(batches[b]))]
    work = [(trees[r::cores], budget_s) for r in range(cores)]
    ctx = mp.get_context("spawn")
    with ctx.Pool(cores) as pool:
        pool.map(_oracle_trees, [([trees[0]], 1.0)] * cores)      # warm the workers (imports)
        t0 = time.perf_counter()
        n = sum(pool.map(_oracle_trees, work))
        dt = time.perf_counter() - t0
    return {"value": n / dt, "unit": "samples/s", "cores": cores, "kind": "oracle", "cpu": lscpu_model(),
            "sample": f"{n} trees of the bench batches in {dt:.1f} s on {cores} processes (FP64 NumPy, "
                      f"BLAS threads = 1 each)"}


def _rank_entry(rank: int, world: int, port: int, argv):
    os.environ.update(RANK=str(rank), LOCAL_RANK=str(rank), WORLD_SIZE=str(world), LOCAL_WORLD_SIZE=str(world),
                      MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    sys.argv = argv
    main()


def spawn_ranks(n: int):
    """`bench.py --gpus N` without torchrun: N processes, one per GPU, as torchrun would start them; each
    times its own steps and rank 0 prints the line with the max over ranks."""
    import socket
    import torch.multiprocessing as mp
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    mp.spawn(_rank_entry, args=(n, port, list(sys.argv)), nprocs=n, join=True)


def lscpu_model() -> str:
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--batch", type=int, default=16)
    ap.add_argument("--impl", default="vpps", choices=["vpps", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-flush", action="store_true")
    ap.add_argument("--groups", type=int, default=4, help="replica groups G (SPEC P1); 148 = 4 x 37")
    ap.add_argument("--cluster", type=int, default=16,
                    help="> 1: whole-graph replica groups of this many CTAs (SPEC S5g)")
    ap.add_argument("--sync", choices=["dataflow", "cluster"], default="dataflow",
                    help="dataflow: epoch-tagged slots, cooperative groups (vpps_df); cluster: hardware "
                         "cluster barrier (vpps_cl)")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)

    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        # launched without torchrun: start the N ranks here (one process per GPU, 127.0.0.1 rendezvous)
        spawn_ranks(args.gpus)
        return
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world != args.gpus:
        sys.exit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world} (launch N ranks with --gpus N)")
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, world, rank)
        return

    import torch
    from paper_conf_micro_khorasanieas18_b200 import vpps

    n_dev = torch.cuda.device_count()
    local = local % n_dev                     # (more ranks than GPUs only in a functional check, see below)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist = None
    backend = "nccl"
    if world > 1:
        import torch.distributed as dist
        # NCCL needs one GPU per rank; ranks sharing a GPU (a functional check of the N-rank path on a
        # smaller box, never a measurement) fall back to gloo and say so in the line
        backend = "nccl" if world <= n_dev else "gloo"
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group("gloo")

    rng = np.random.default_rng(1234)          # identical initial parameters on every rank
    shapes = vpps.param_shapes("binary", H, E, C)
    P = synth.init_params(shapes, rng)
    X = synth.input_table(rng, V, E)
    m = vpps.Model("binary", H, E, C, device=local, groups=args.groups, cluster=args.cluster,
                   dataflow=bool(args.cluster) and args.sync == "dataflow")
    params = torch.zeros(m.n_floats, dtype=torch.float32, device=dev)
    grads = torch.zeros_like(params)
    for name, _ in shapes:
        m.views(params)[name].copy_(torch.from_numpy(P[name]).float())
    m.bind(params, grads)
    inputs = torch.from_numpy(X).float().to(dev)
    d_inputs = torch.zeros_like(inputs)
    stream = torch.cuda.current_stream()
    batches = make_batches(rank, args.batch)
    scripts = [m.build_script(g) for g in batches]
    for s in scripts:
        s.upload()
    infos = [s.info() for s in scripts]
    flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device=dev)   # 256 MiB > 126 MB L2
    flush2 = torch.ones(64 * 1024 * 1024, dtype=torch.float32, device=dev) if os.environ.get("VPPS_FLUSH_CLEAN") else None
    lr, wd = 1e-3, 1e-5

    from paper_conf_micro_khorasanieas18_b200 import dp

    def step(k):
        s = scripts[k % N_BATCHES]
        if world == 1:
            m.fwd_bwd_sgd(s, inputs, d_inputs, lr=lr, weight_decay=wd)
        else:
            dp.dp_step(m, s, inputs, d_inputs, grads, lr, wd)

    kb, ka = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for w in range(args.warmup):
        step(w)
    torch.cuda.synchronize()
    if dist:
        dist.barrier()
    torch.cuda.synchronize()

    clocks = ClockSampler(local)
    clocks.start()
    step_ms, kern_ms, flops = 0.0, 0.0, 0.0
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    kev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    for a, b in kev:            # torch creates the CUDA event lazily on first record
        a.record(stream)
        b.record(stream)
    torch.cuda.synchronize()
    for k in range(args.steps):
        if not args.no_flush:
            flush.zero_()
            if os.environ.get("VPPS_FLUSH_CLEAN"):     # measurement experiment: leave the L2 clean
                flush2.sum()
        m.set_timing_events(*kev[k])
        ev[k][0].record(stream)
        step(args.warmup + k)
        ev[k][1].record(stream)
        flops += infos[(args.warmup + k) % N_BATCHES]["flops"]
    m.set_timing_events(None, None)
    # north_star roofline per batch: T = max(F / P_fp32, (2 W_once + A) / BW_HBM), averaged over the timed
    # batches (F, A: the script's algorithmic FLOPs and activation bytes)
    torch.cuda.synchronize()
    clk = clocks.stop()
    step_ms = sum(a.elapsed_time(b) for a, b in ev)
    kern_ms = sum(a.elapsed_time(b) for a, b in kev)
    t = torch.tensor([step_ms, kern_ms], dtype=torch.float64, device=dev)
    if dist:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    step_ms, kern_ms = float(t[0]), float(t[1])

    # ---- dominant kernel alone (vpps_df / vpps_cl): CUDA events recorded around it on the launching
    #      stream.  The records break the programmatic overlap with the neighbouring GEMMs, so this is a
    #      separate pass, not the timed region above ----
    dom_ms, dom_flops, dom_n = 0.0, 0.0, 0
    if args.cluster:
        kd = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
              for _ in range(min(args.steps, 100))]
        for a, b in kd:
            a.record(stream)
            b.record(stream)
        torch.cuda.synchronize()
        for k, (a, b) in enumerate(kd):
            if not args.no_flush:
                flush.zero_()
            m.set_kernel_events(a, b)
            step(args.warmup + k)
            dom_flops += infos[(args.warmup + k) % N_BATCHES]["kernel_flops"]
        m.set_kernel_events(None, None)
        torch.cuda.synchronize()
        dom_n = len(kd)
        dom_ms = sum(a.elapsed_time(b) for a, b in kd)
        t = torch.tensor([dom_ms], dtype=torch.float64, device=dev)
        if dist:
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dom_ms = float(t[0])

    # ---- end to end through the public API: host script build + one H2D copy + kernel + loss D2H ----
    e2e_steps = min(args.steps, 200)
    h2d = 0
    csr = [vpps.CsrBatch.from_graphs(g) for g in batches]   # the data loader's output: CSR batches (API input)
    from concurrent.futures import ThreadPoolExecutor
    builders = ThreadPoolExecutor(max_workers=3)            # the data loader's worker pool, started up front
    for k, s in enumerate(vpps.prefetch_scripts(m, (csr[(k + 7) % N_BATCHES] for k in range(args.warmup)),
                                                executor=builders)):
        m.fwd_bwd_sgd(s, inputs, d_inputs, lr=lr, weight_decay=wd) if world == 1 else \
            dp.dp_step(m, s, inputs, d_inputs, grads, lr, wd)     # untimed: warms builders and staging ring
    m.latest_loss()
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    # host: super-graph, levels, schedule, encode — built a few batches ahead by 3 background workers
    for k, s in enumerate(vpps.prefetch_scripts(m, (csr[k % N_BATCHES] for k in range(e2e_steps)),
                                                executor=builders)):
        h2d += s.info()["blob_words"] * 4            # staged by the call below: one pinned H2D copy (L169)
        if world == 1:
            m.fwd_bwd_sgd(s, inputs, d_inputs, lr=lr, weight_decay=wd)
        else:
            dp.dp_step(m, s, inputs, d_inputs, grads, lr, wd)
        if k > 0:
            m.stale_loss()                           # D2H'd loss of the previous step (PAPER's stale loss)
    m.latest_loss()                                  # the last step's loss
    torch.cuda.synchronize()
    e2e_s = time.perf_counter() - t0
    builders.shutdown()
    te = torch.tensor([e2e_s], dtype=torch.float64, device=dev)
    if dist:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_s = float(te[0])

    if rank == 0:
        samples = args.steps * args.batch * world
        value = samples / (step_ms / 1e3)
        pk = peaks()
        mhz = clk.get("sm_mhz") or pk.get("sm_max_mhz", 1965.0)
        peak = fp32_peak_tflops(pk.get("sm_max_mhz", 1965.0))
        try:
            bw_hbm = float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]) * 1e9
        except Exception:
            bw_hbm = 7.7e12                                  # B200_PROFILING.md fallback
        w_once_b = 4 * sum(int(np.prod(s)) for _, s in shapes)
        t_roof = [max(inf["flops"] / (peak * 1e12), (2 * w_once_b + inf["act_bytes"]) / bw_hbm)
                  for inf in (infos[(args.warmup + k) % N_BATCHES] for k in range(args.steps))]
        t_roof_mean = float(np.mean(t_roof))
        avg_flops = flops / args.steps
        step_tflops = avg_flops / (kern_ms / args.steps / 1e3) / 1e12
        if dom_n:
            dom_avg_ms = dom_ms / dom_n
            dom_avg_flops = dom_flops / dom_n
            achieved = dom_avg_flops / (dom_avg_ms / 1e3) / 1e12
        else:
            dom_avg_ms, dom_avg_flops, achieved = kern_ms / args.steps, avg_flops, step_tflops
        w_once = 4 * sum(int(np.prod(s)) for _, s in shapes if len(s) == 2)
        traffic = inpipe = None
        prof = os.path.join(ROOT, "profiles", f"{PROFILE_TAG}_ncu_summary.json")
        if os.path.exists(prof):
            try:
                pj = json.load(open(prof))
                traffic = pj.get("dram_bytes_per_launch")
                inpipe = pj.get("in_pipeline")
            except Exception:
                traffic = inpipe = None
        line = {
            "metric": METRIC, "value": value, "unit": "samples/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": step_ms / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "impl": "vpps",
            "config": {"workload": WORKLOAD, "global_batch": args.batch * world, "per_gpu_batch": args.batch,
                       "seq_len": None, "parallelism": f"dp{world}",
                       "backend": backend if world > 1 else None,
                       "replica_groups": m.plan_info()["n_cta"] // m.plan_info()["n_g"],
                       "cluster": args.cluster or None, "ctas": m.plan_info()["n_cta"],
                       "sync": (args.sync if args.cluster else "grid barrier"),
                       "mode": ("leaf GEMM + replica-group fwd/bwd + dW/dX GEMM + SGD" if args.cluster
                                else "fused fwd-bwd-sgd, 1 kernel") + ("" if world == 1 else ", NCCL all-reduce before SGD"),
                       "l2": "no flush" if args.no_flush else "flushed (256 MiB write) before every timed step",
                       "batches": f"{N_BATCHES} distinct pre-built scripts cycled"},
            # leaf GEMM + vpps_df + gradient GEMM (SGD fused in its tail at N = 1; a separate sgd_kernel after
            # the all-reduce at N > 1); the grid path: one fused kernel (+ sgd_kernel at N > 1)
            "gpu_launches": args.steps * ((3 if world == 1 else 4) if args.cluster else (1 if world == 1 else 2)),
            "roofline": {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "TFLOP/s",
                         "frac": achieved / peak, "traffic": traffic,
                         "kernel": ("vpps_df" if args.sync == "dataflow" else "vpps_cl") if args.cluster else "vpps_fb",
                         "kernel_ms": dom_avg_ms, "flops_per_launch": dom_avg_flops,
                         "step_kernels_ms": kern_ms / args.steps, "step_flops": avg_flops,
                         "step_tflops": step_tflops,
                         "peak_note": "FP32 FFMA: 148 SM x 128 lanes x 2 FLOP x sm_max_mhz (derived, DESIGN.md)",
                         "north_star": {"t_roofline_us": 1e6 * t_roof_mean,
                                        "t_measured_us": 1e3 * step_ms / args.steps,
                                        "frac": 1e6 * t_roof_mean / (1e3 * step_ms / args.steps),
                                        "definition": "max(F / P_fp32, (2 W_once + A) / BW_hbm) per batch, "
                                                      "mean over the timed batches, / measured step time"}},
            "dram": {"weights_once_bytes": w_once,
                     "dominant_kernel_cold_bytes": traffic,
                     "pass_read_bytes_in_pipeline": inpipe["pass_dram_read_bytes"] if inpipe else None,
                     "pass_read_vs_weights_once": (inpipe["pass_dram_read_bytes"] / w_once) if inpipe else None,
                     "pass_write_bytes_in_pipeline": inpipe["pass_dram_write_bytes"] if inpipe else None,
                     "note": "cold: ncu --set full of the dominant kernel (caches flushed per replay); in pipeline: "
                             "ncu --cache-control none over bench steps, all kernels of a pass (writes include "
                             "evictions of the L2-flush buffer's dirty lines)",
                     "source": f"profiles/{PROFILE_TAG}_ncu_summary.json" if traffic else None},
            "e2e": {"value": e2e_steps * args.batch * world / e2e_s, "unit": "samples/s",
                    "h2d_bytes_per_step": h2d // e2e_steps, "d2h_bytes_per_step": 4,
                    "includes": "per step: host script build from the step's CSR batch (3 builder threads, 4 ahead) + pinned H2D copy of the script + kernels (+ all-reduce) + loss D2H (stale-loss read); CSR batches are the data loader's output, made before the timed region"},
            "clocks": clk,
        }
        if world == 1 and not args.no_cpu_baseline:
            line["cpu_baseline"] = cpu_baseline(batches)
            line["cpu_baseline_all_cores"] = cpu_baseline_all_cores(batches)
        print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
