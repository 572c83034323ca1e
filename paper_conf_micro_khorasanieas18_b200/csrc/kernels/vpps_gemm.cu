// Dense FP32 products of the level-synchronous path (sm_100a): the per-level / per-step concatenated
// products and the per-matrix gradient GEMMs of PAPER L185 ("concatenate all the left hand side and all
// the right hand side tensors ... and use dense matrix-matrix multiplication").  Hand-written SIMT FFMA2
// tiles replace the library SGEMM the path used before; plain FP32 (no TF32 / emulation: R-22's 1e-4).
//
// C[M x N] = op(A) op(B) + beta C, row-major; op(A)(m, k) = TA ? A[k lda + m] : A[m lda + k],
// op(B)(k, n) = TB ? B[n ldb + k] : B[k ldb + n].
//
// Tiles of BM x BN outputs per CTA, K in steps of BK = 16 staged k-major in shared memory (both operands
// transposed on the way in when they are contiguous along k), register double buffering (the next k-step
// is loaded while the current one is computed, one barrier per k-step), TM x TN outputs per thread as
// FFMA2 pairs.  Shapes with few tiles are split along K; the split CTAs add their partial tiles into C
// with red.global.add (C cleared first when beta = 0).
#include <algorithm>
#include <cstdint>
#include <cuda_runtime.h>

#include "vpps_kernel.cuh"

namespace vpps {
namespace dev {
namespace gm {

constexpr int BK = 16;

template <int BM, int BN, int TM, int TN>
struct Tile {
    static constexpr int NT = (BM / TM) * (BN / TN);   // threads
    static constexpr int PA = BM + 4, PB = BN + 4;       // padded k-major rows
    static constexpr int LA = BM * BK / NT;              // A elements loaded per thread per k-step
    static constexpr int LB = BN * BK / NT;
    static_assert(TM == 4 || TM == 8, "TM");
    static_assert(TN == 4 || TN == 8, "TN");
    static_assert(LA % 4 == 0 && LB % 4 == 0, "whole float4 groups per thread");
};

// one k-step of an operand into registers: R elements as R/4 groups of 4 consecutive elements along the
// operand's contiguous dimension.  KC = the operand is contiguous along k (A not transposed, B transposed).
template <bool KC, int ROWS, int NT, int R, bool VEC>
__device__ __forceinline__ void load_step(const float* __restrict__ X, int ld, int r0, int rmax, int k0, int kmax,
                                          float (&v)[R]) {
#pragma unroll
    for (int i = 0; i < R / 4; ++i) {
        const int g = threadIdx.x + i * NT;
        int r, k;
        if (KC) { r = g / (BK / 4); k = (g % (BK / 4)) * 4; }      // 4 consecutive k of row r
        else { k = g / (ROWS / 4); r = (g % (ROWS / 4)) * 4; }     // 4 consecutive rows at k
        const int gr = r0 + r, gk = k0 + k;
        const bool full = KC ? (gr < rmax && gk + 3 < kmax) : (gk < kmax && gr + 3 < rmax);
        if (VEC && full) {
            const float4 x = __ldg(reinterpret_cast<const float4*>(KC ? X + (int64_t)gr * ld + gk
                                                                      : X + (int64_t)gk * ld + gr));
            v[4 * i] = x.x; v[4 * i + 1] = x.y; v[4 * i + 2] = x.z; v[4 * i + 3] = x.w;
        } else {
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int rr = KC ? gr : gr + q, kk = KC ? gk + q : gk;
                v[4 * i + q] = (rr < rmax && kk < kmax) ? __ldg(X + (KC ? (int64_t)rr * ld + kk : (int64_t)kk * ld + rr)) : 0.f;
            }
        }
    }
}

// the registers of one k-step into the k-major shared tile S[BK][P]
template <bool KC, int ROWS, int NT, int R, int P>
__device__ __forceinline__ void store_step(float* S, const float (&v)[R]) {
#pragma unroll
    for (int i = 0; i < R / 4; ++i) {
        const int g = threadIdx.x + i * NT;
        if (KC) {
            const int r = g / (BK / 4), k = (g % (BK / 4)) * 4;
#pragma unroll
            for (int q = 0; q < 4; ++q) S[(k + q) * P + r] = v[4 * i + q];
        } else {
            const int k = g / (ROWS / 4), r = (g % (ROWS / 4)) * 4;
            *reinterpret_cast<float4*>(S + k * P + r) = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
        }
    }
}

template <bool TA, bool TB, bool VEC, int BM, int BN, int TM, int TN>
__global__ void __launch_bounds__(Tile<BM, BN, TM, TN>::NT, 2)
sgemm(int M, int N, int K, const float* __restrict__ A, int lda, const float* __restrict__ B, int ldb,
      float* __restrict__ C, int ldc, float beta, int k_split) {
    using T = Tile<BM, BN, TM, TN>;
    constexpr int NT = T::NT, PA = T::PA, PB = T::PB;
    __shared__ __align__(16) float As[2][BK * PA];
    __shared__ __align__(16) float Bs[2][BK * PB];
    const int m0 = blockIdx.y * BM, n0 = blockIdx.x * BN;
    const int kb = blockIdx.z * k_split, ke = min(K, kb + k_split);
    const int tid = threadIdx.x;
    const int ty = tid / (BN / TN), tx = tid % (BN / TN);

    float2 acc[TM][TN / 2];
#pragma unroll
    for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN / 2; ++j) acc[i][j] = make_float2(0.f, 0.f);

    float ra[T::LA], rb[T::LB];
    // A: rows m contiguous along k unless TA;  B: rows n contiguous along k iff TB
    load_step<!TA, BM, NT, T::LA, VEC>(A, lda, m0, M, kb, ke, ra);
    load_step<TB, BN, NT, T::LB, VEC>(B, ldb, n0, N, kb, ke, rb);
    store_step<!TA, BM, NT, T::LA, PA>(As[0], ra);
    store_step<TB, BN, NT, T::LB, PB>(Bs[0], rb);
    __syncthreads();
    int cur = 0;
    for (int k0 = kb; k0 < ke; k0 += BK) {
        const bool more = k0 + BK < ke;
        if (more) {
            load_step<!TA, BM, NT, T::LA, VEC>(A, lda, m0, M, k0 + BK, ke, ra);
            load_step<TB, BN, NT, T::LB, VEC>(B, ldb, n0, N, k0 + BK, ke, rb);
        }
        const float* as = As[cur];
        const float* bs = Bs[cur];
#pragma unroll
        for (int k = 0; k < BK; ++k) {
            float a[TM], b[TN];
#pragma unroll
            for (int h = 0; h < TM / 4; ++h) {
                const float4 x = *reinterpret_cast<const float4*>(as + k * PA + h * (BM / 2) + ty * 4);
                a[4 * h] = x.x; a[4 * h + 1] = x.y; a[4 * h + 2] = x.z; a[4 * h + 3] = x.w;
            }
#pragma unroll
            for (int h = 0; h < TN / 4; ++h) {
                const float4 x = *reinterpret_cast<const float4*>(bs + k * PB + h * (BN / 2) + tx * 4);
                b[4 * h] = x.x; b[4 * h + 1] = x.y; b[4 * h + 2] = x.z; b[4 * h + 3] = x.w;
            }
#pragma unroll
            for (int i = 0; i < TM; ++i)
#pragma unroll
                for (int j = 0; j < TN / 2; ++j)
                    acc[i][j] = __ffma2_rn(make_float2(a[i], a[i]), make_float2(b[2 * j], b[2 * j + 1]), acc[i][j]);
        }
        if (more) {
            store_step<!TA, BM, NT, T::LA, PA>(As[cur ^ 1], ra);
            store_step<TB, BN, NT, T::LB, PB>(Bs[cur ^ 1], rb);
        }
        __syncthreads();
        cur ^= 1;
    }
    // epilogue: thread rows m = m0 + h (BM/2) + 4 ty + i, columns n = n0 + h (BN/2) + 4 tx + j
    const bool split = gridDim.z > 1;
#pragma unroll
    for (int i = 0; i < TM; ++i) {
        const int m = m0 + (i / 4) * (BM / 2) + ty * 4 + (i % 4);
        if (m >= M) continue;
        float* crow = C + (int64_t)m * ldc;
#pragma unroll
        for (int j = 0; j < TN / 2; ++j) {
            const int n = n0 + ((2 * j) / 4) * (BN / 2) + tx * 4 + (2 * j) % 4;
            const float v0 = acc[i][j].x, v1 = acc[i][j].y;
            if (split) {
                if (n < N) atomicAdd(crow + n, v0);
                if (n + 1 < N) atomicAdd(crow + n + 1, v1);
            } else if (beta == 0.f) {
                if (n < N) crow[n] = v0;
                if (n + 1 < N) crow[n + 1] = v1;
            } else {
                if (n < N) crow[n] = v0 + beta * crow[n];
                if (n + 1 < N) crow[n + 1] = v1 + beta * crow[n + 1];
            }
        }
    }
}

template <int BM, int BN, int TM, int TN, bool TA, bool TB>
cudaError_t launch_cfg(bool vec, int M, int N, int K, const float* A, int lda, const float* B, int ldb, float* C,
                       int ldc, float beta, cudaStream_t s) {
    constexpr int NT = Tile<BM, BN, TM, TN>::NT;
    const int tm = (M + BM - 1) / BM, tn = (N + BN - 1) / BN, tiles = tm * tn;
    // split K when the tiles alone do not fill the GPU twice over (every split keeps >= 4 k-steps)
    int splits = 1;
    if (tiles < 2 * 148 && K >= 8 * BK)
        splits = std::max(1, std::min((2 * 148 + tiles - 1) / tiles, K / (4 * BK)));
    int k_split = (K + splits - 1) / splits;
    k_split = (k_split + BK - 1) / BK * BK;
    splits = (K + k_split - 1) / k_split;
    if (splits > 1) {
        if (beta == 0.f) {
            // the partial tiles are summed into C: clear it first (row by row when ldc > N)
            cudaError_t e = ldc == N ? cudaMemsetAsync(C, 0, (size_t)M * N * sizeof(float), s)
                                     : cudaMemset2DAsync(C, (size_t)ldc * sizeof(float), 0, (size_t)N * sizeof(float), M, s);
            if (e != cudaSuccess) return e;
        } else if (beta != 1.f) {
            return cudaErrorInvalidValue;     // (the level path uses beta 0 or 1)
        }
    }
    const dim3 grid(tn, tm, splits);
    if (vec) sgemm<TA, TB, true, BM, BN, TM, TN><<<grid, NT, 0, s>>>(M, N, K, A, lda, B, ldb, C, ldc, beta, k_split);
    else sgemm<TA, TB, false, BM, BN, TM, TN><<<grid, NT, 0, s>>>(M, N, K, A, lda, B, ldb, C, ldc, beta, k_split);
    return cudaGetLastError();
}

template <bool TA, bool TB>
cudaError_t dispatch(int M, int N, int K, const float* A, int lda, const float* B, int ldb, float* C, int ldc,
                     float beta, cudaStream_t s) {
    const bool vec = lda % 4 == 0 && ldb % 4 == 0 && ((uintptr_t)A & 15) == 0 && ((uintptr_t)B & 15) == 0;
    const int64_t t128 = (int64_t)((M + 127) / 128) * ((N + 127) / 128);
    if (M >= 128 && N >= 128 && t128 >= 148)
        return launch_cfg<128, 128, 8, 8, TA, TB>(vec, M, N, K, A, lda, B, ldb, C, ldc, beta, s);
    if (M > 32)
        return launch_cfg<64, 64, 4, 4, TA, TB>(vec, M, N, K, A, lda, B, ldb, C, ldc, beta, s);
    if (M > 16)
        return launch_cfg<32, 64, 4, 4, TA, TB>(vec, M, N, K, A, lda, B, ldb, C, ldc, beta, s);
    return launch_cfg<16, 64, 4, 4, TA, TB>(vec, M, N, K, A, lda, B, ldb, C, ldc, beta, s);
}

}  // namespace gm
}  // namespace dev

cudaError_t gemm_f32(cudaStream_t s, bool ta, bool tb, int M, int N, int K, const float* A, int lda, const float* B,
                     int ldb, float* C, int ldc, float beta) {
    using namespace dev::gm;
    if (M <= 0 || N <= 0) return cudaSuccess;
    if (K <= 0) {       // an empty sum: C = beta C (only dW products of node-less levels: beta = 0)
        if (beta != 0.f) return cudaSuccess;
        return ldc == N ? cudaMemsetAsync(C, 0, (size_t)M * N * sizeof(float), s)
                        : cudaMemset2DAsync(C, (size_t)ldc * sizeof(float), 0, (size_t)N * sizeof(float), M, s);
    }
    if (!ta && tb) return dispatch<false, true>(M, N, K, A, lda, B, ldb, C, ldc, beta, s);
    if (!ta && !tb) return dispatch<false, false>(M, N, K, A, lda, B, ldb, C, ldc, beta, s);
    if (ta && !tb) return dispatch<true, false>(M, N, K, A, lda, B, ldb, C, ldc, beta, s);
    return dispatch<true, true>(M, N, K, A, lda, B, ldb, C, ldc, beta, s);
}

}  // namespace vpps

// C ABI (include/vpps.h): the level path's dense product, exposed for direct testing
extern "C" int32_t vpps_gemm_f32(void* stream, int32_t ta, int32_t tb, int32_t M, int32_t N, int32_t K, const float* A,
                                 int32_t lda, const float* B, int32_t ldb, float* C, int32_t ldc, float beta) {
    if (M < 0 || N < 0 || K < 0 || (beta != 0.f && beta != 1.f) || (M > 0 && N > 0 && (!C || (K > 0 && (!A || !B)))))
        return -1;   // VPPS_E_INVALID
    return vpps::gemm_f32((cudaStream_t)stream, ta != 0, tb != 0, M, N, K, A, lda, B, ldb, C, ldc, beta) == cudaSuccess
               ? 0 : -3;   // VPPS_E_CUDA
}
