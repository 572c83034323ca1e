"""Throughput of vpps_gemm_f32 (the level paths' dense product) on a few shapes, CUDA-event timed.
    VPPS_GEMM_TC_MIN=-1 python tools/gemm_bench.py     (FFMA2 tiles only)"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_micro_khorasanieas18_b200 import vpps  # noqa: E402

SHAPES = [(4096, 4096, 4096, False, True), (3072, 2048, 1700, True, False), (1000, 3072, 2048, False, True),
          (1000, 2048, 3072, False, False), (768, 512, 424, True, False), (128, 128, 4096, False, True)]
for M, N, K, ta, tb in SHAPES:
    A = torch.randn((K, M) if ta else (M, K), device="cuda")
    B = torch.randn((N, K) if tb else (K, N), device="cuda")
    C = torch.zeros(M, N, device="cuda")
    for _ in range(3):
        vpps.gemm_f32(A, B, C, ta=ta, tb=tb)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    n = 20
    e0.record()
    for _ in range(n):
        vpps.gemm_f32(A, B, C, ta=ta, tb=tb)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / n
    print(f"M={M} N={N} K={K} ta={int(ta)} tb={int(tb)}: {ms*1e3:8.1f} us  {2*M*N*K/ms/1e9:7.1f} TFLOP/s")
