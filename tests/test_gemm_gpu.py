"""The level paths' dense FP32 product (csrc/kernels/vpps_gemm.cu) against float64 torch
matmuls: every transpose combination, every tile configuration (M from 1 to 3072), ragged edges, unaligned
leading dimensions (scalar loads), split-K with beta 0 and 1, and K = 0.  Bound: |C - C64| <= 1e-5 ·
(|A| |B|)(m, n) + tiny (an FP32 sum of K products)."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

SHAPES = [(1, 5, 7), (3, 9, 1000), (16, 2048, 512), (17, 1024, 256), (33, 3072, 2048), (64, 1000, 256),
          (100, 300, 40), (128, 128, 16), (500, 1024, 257), (1000, 3072, 2048), (3072, 2048, 1700), (768, 512, 64),
          (9, 256, 2240), (256, 9, 2240)]


def _ref(A, B, C0, ta, tb, beta):
    a = A.double().t() if ta else A.double()
    b = B.double().t() if tb else B.double()
    return a @ b + beta * C0.double(), a.abs() @ b.abs()


@pytest.mark.parametrize("ta,tb", [(False, True), (False, False), (True, False), (True, True)])
@pytest.mark.parametrize("shape", SHAPES)
def test_gemm_against_float64(ta, tb, shape):
    from paper_conf_micro_khorasanieas18_b200 import vpps
    M, N, K = shape
    g = torch.Generator(device="cuda").manual_seed(M * 7 + N * 3 + K)
    A = torch.randn((K, M) if ta else (M, K), device="cuda", generator=g)
    B = torch.randn((N, K) if tb else (K, N), device="cuda", generator=g)
    for beta in (0.0, 1.0):
        C = torch.randn(M, N, device="cuda", generator=g)
        C0 = C.clone()
        vpps.gemm_f32(A, B, C, ta=ta, tb=tb, beta=beta)
        torch.cuda.synchronize()
        ref, mag = _ref(A, B, C0, ta, tb, beta)
        err = (C.double() - ref).abs()
        assert bool((err <= 1e-5 * mag + 1e-5 * C0.double().abs() * beta + 1e-30).all()), (shape, beta, float(err.max()))


def test_gemm_strided_and_unaligned():
    """Leading dimensions larger than the row (sub-blocks of a wider buffer, as the level path's Z / G
    buffers), odd leading dimensions and a K = 0 product (C = 0 when beta = 0)."""
    from paper_conf_micro_khorasanieas18_b200 import vpps
    g = torch.Generator(device="cuda").manual_seed(5)
    W = torch.randn(40, 37, device="cuda", generator=g)      # odd ld: unaligned rows
    X = torch.randn(23, 37, device="cuda", generator=g)
    Z = torch.zeros(23, 101, device="cuda")
    vpps.gemm_f32(X, W, Z, tb=True, M=23, N=40, K=37, ldc=101)
    torch.cuda.synchronize()
    ref = X.double() @ W.double().t()
    assert float((Z[:, :40].double() - ref).abs().max()) <= 1e-5 * float((X.abs().double() @ W.abs().double().t()).max())
    assert float(Z[:, 40:].abs().max()) == 0.0
    C = torch.ones(8, 8, device="cuda")
    vpps.gemm_f32(X, W, C, M=8, N=8, K=0)
    torch.cuda.synchronize()
    assert float(C.abs().max()) == 0.0


TC_SHAPES = [(64, 64, 64), (65, 129, 70), (200, 96, 100), (128, 128, 4096), (300, 1000, 257), (1000, 3072, 2048)]


@pytest.mark.parametrize("mode", ["0", "-1"])
def test_gemm_tensor_core_and_simt_forced(mode):
    """VPPS_GEMM_TC_MIN=0 sends every product with M, N, K >= 64 to the tcgen05 3xTF32 tiles (ragged tiles,
    split-K, all transposes, beta 0 / 1); -1 keeps every product on the FFMA2 tiles.  The switch is read
    once per process, so each mode runs in a child process."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = ("import sys; sys.path.insert(0, %r); sys.path.insert(0, %r); import test_gemm_gpu as t\n"
            "for ta in (False, True):\n"
            "  for tb in (False, True):\n"
            "    for sh in t.TC_SHAPES + t.SHAPES[:6]:\n"
            "      t.test_gemm_against_float64(ta, tb, sh)\n"
            "print('ok')" % (root, os.path.join(root, "tests")))
    r = subprocess.run([sys.executable, "-c", code], env={**os.environ, "VPPS_GEMM_TC_MIN": mode}, capture_output=True,
                       text=True, timeout=900)
    assert r.returncode == 0 and "ok" in r.stdout, r.stdout + r.stderr
