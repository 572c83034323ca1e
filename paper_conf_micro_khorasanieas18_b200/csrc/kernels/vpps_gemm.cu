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
#include <atomic>
#include <cstdlib>
#include <cuda_runtime.h>

#include "dev_common.cuh"
#include "tc_common.cuh"
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

// ---- tensor-core tiles: tcgen05.mma kind::tf32 with a 3xTF32 split (FP32 accuracy; tc_common.cuh) --------
// Large products (the C5-sized level products and per-matrix gradient GEMMs: a level batches enough
// same-parameter nodes to form a real dense GEMM, north_star) run on the 5th-gen tensor cores: D[128 x 128]
// per CTA in TMEM, K in chunks of 32 through two register-staged stages; the loads of chunk c + 1 are in
// flight while chunk c is converted and multiplied.
namespace tc {
using namespace tcc;

// one operand's share of a chunk (piece_rk): 16-byte global loads along the operand's contiguous dimension
template <bool KC>
__device__ __forceinline__ void load_chunk(const float* __restrict__ X, int ld, int r0, int rmax, int k0, int kmax,
                                           float4 (&v)[4]) {
#pragma unroll
    for (int p = 0; p < 4; ++p) {
        int r, k;
        piece_rk(KC, p, r, k);
        const int gr = r0 + r, gk = k0 + k;
        float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
        if (KC) {
            if (gr < rmax) {
                const float* src = X + (int64_t)gr * ld + gk;
                if (gk + 3 < kmax) x = __ldg(reinterpret_cast<const float4*>(src));
                else {
                    if (gk < kmax) x.x = __ldg(src);
                    if (gk + 1 < kmax) x.y = __ldg(src + 1);
                    if (gk + 2 < kmax) x.z = __ldg(src + 2);
                }
            }
        } else if (gk < kmax) {
            const float* src = X + (int64_t)gk * ld + gr;
            if (gr + 3 < rmax) x = __ldg(reinterpret_cast<const float4*>(src));
            else {
                if (gr < rmax) x.x = __ldg(src);
                if (gr + 1 < rmax) x.y = __ldg(src + 1);
                if (gr + 2 < rmax) x.z = __ldg(src + 2);
            }
        }
        v[p] = x;
    }
}

template <bool TA, bool TB>
__global__ void __launch_bounds__(NT, 1)
tc_sgemm(int M, int N, int K, const float* __restrict__ A, int lda, const float* __restrict__ B, int ldb,
         float* __restrict__ C, int ldc, float beta, int k_split) {
    extern __shared__ __align__(128) float tsm[];
    __shared__ uint32_t tmem_base;
    __shared__ __align__(8) uint64_t mbar[2];
    float* sm = reinterpret_cast<float*>((reinterpret_cast<uintptr_t>(tsm) + 127) & ~uintptr_t(127));
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const int m0 = blockIdx.y * BM, n0 = blockIdx.x * BN;
    const int kb = blockIdx.z * k_split, ke = min(K, kb + k_split);
    const int nch = (ke - kb + BKC - 1) / BKC;
    float4 ra[4], rb[4];
    load_chunk<!TA>(A, lda, m0, M, kb, ke, ra);
    load_chunk<TB>(B, ldb, n0, N, kb, ke, rb);
    setup(&tmem_base, mbar);
    const uint32_t tmem = tmem_base;
    uint32_t phases = 0u;                          // bit st: parity of stage st's next completion
    for (int c = 0; c < nch; ++c) {
        const int st = c & 1;
        float* Ah = sm + st * STAGE_F;
        if (c >= 2) { mbar_wait(smem_u32(&mbar[st]), (phases >> st) & 1u); phases ^= 1u << st; }   // chunk c - 2 read it
        store_chunk<!TA>(Ah, Ah + OP_F, ra);
        store_chunk<TB>(Ah + 2 * OP_F, Ah + 3 * OP_F, rb);
        if (c + 1 < nch) {                        // next chunk's loads in flight during this chunk's MMAs
            load_chunk<!TA>(A, lda, m0, M, kb + (c + 1) * BKC, ke, ra);
            load_chunk<TB>(B, ldb, n0, N, kb + (c + 1) * BKC, ke, rb);
        }
        issue_chunk(tmem, Ah, &mbar[st], c == 0);
    }
    if (nch > 0) {                                 // the last commit covers every earlier MMA
        const int st = (nch - 1) & 1;
        mbar_wait(smem_u32(&mbar[st]), (phases >> st) & 1u);
    }
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    // epilogue: warp w holds rows 32 (w & 3) + lane, columns 64 (w >> 2) .. +63
    const int row = m0 + 32 * (warp & 3) + lane, cb = 64 * (warp >> 2);
    const bool split = gridDim.z > 1;
    const bool vec = (ldc & 3) == 0 && ((reinterpret_cast<uintptr_t>(C) & 15) == 0);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        uint32_t r[16];
        load16(tmem, cb + 16 * q, r);
        if (nch == 0)
#pragma unroll
            for (int j = 0; j < 16; ++j) r[j] = 0u;
        if (row < M) {
            float* crow = C + (int64_t)row * ldc + n0 + cb + 16 * q;
            const int nleft = N - (n0 + cb + 16 * q);
#pragma unroll
            for (int j = 0; j < 16; j += 4) {
                const float4 d = make_float4(__uint_as_float(r[j]), __uint_as_float(r[j + 1]), __uint_as_float(r[j + 2]),
                                             __uint_as_float(r[j + 3]));
                if (vec && j + 3 < nleft) {
                    if (split) red_add<4>(crow + j, &d.x);
                    else if (beta == 0.f) *reinterpret_cast<float4*>(crow + j) = d;
                    else {
                        const float4 o = *reinterpret_cast<const float4*>(crow + j);
                        *reinterpret_cast<float4*>(crow + j) = make_float4(d.x + o.x, d.y + o.y, d.z + o.z, d.w + o.w);
                    }
                } else {
                    const float e[4] = {d.x, d.y, d.z, d.w};
#pragma unroll
                    for (int t = 0; t < 4; ++t) {
                        if (j + t >= nleft) break;
                        if (split) atomicAdd(crow + j + t, e[t]);
                        else crow[j + t] = e[t] + (beta == 0.f ? 0.f : crow[j + t]);
                    }
                }
            }
        }
    }
    teardown(tmem);
}

template <bool TA, bool TB>
cudaError_t launch(int M, int N, int K, const float* A, int lda, const float* B, int ldb, float* C, int ldc, float beta,
                   cudaStream_t s) {
    static_assert(SMEM <= 227 * 1024, "stages fit");
    // the dynamic shared memory attribute, once per device (idempotent; a race only repeats it)
    static std::atomic<uint64_t> attr_done{0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (!(attr_done.load() >> (dev & 63) & 1)) {
        const cudaError_t e = cudaFuncSetAttribute(tc_sgemm<TA, TB>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM);
        if (e != cudaSuccess) return e;
        attr_done.fetch_or(uint64_t(1) << (dev & 63));
    }
    const int tm = (M + BM - 1) / BM, tn = (N + BN - 1) / BN, tiles = tm * tn;
    int splits = 1;
    if (tiles < 148 && K >= 8 * BKC) splits = std::max(1, std::min((148 + tiles - 1) / tiles, K / (4 * BKC)));
    int k_split = (K + splits - 1) / splits;
    k_split = (k_split + BKC - 1) / BKC * BKC;
    splits = (K + k_split - 1) / k_split;
    if (splits > 1 && beta == 0.f) {
        cudaError_t e = ldc == N ? cudaMemsetAsync(C, 0, (size_t)M * N * sizeof(float), s)
                                 : cudaMemset2DAsync(C, (size_t)ldc * sizeof(float), 0, (size_t)N * sizeof(float), M, s);
        if (e != cudaSuccess) return e;
    }
    tc_sgemm<TA, TB><<<dim3(tn, tm, splits), NT, SMEM, s>>>(M, N, K, A, lda, B, ldb, C, ldc, beta, k_split);
    return cudaGetLastError();
}
}  // namespace tc

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

// products of at least this many MACs (and >= 64 rows / columns / k) run on the tensor cores
static int64_t g_tc_min_macs = -2;
static int64_t tc_min_macs() {
    if (g_tc_min_macs == -2) {
        const char* e = getenv("VPPS_GEMM_TC_MIN");            // measurement knob; -1 disables the TC tiles
        g_tc_min_macs = e ? atoll(e) : (int64_t)1 << 26;
    }
    return g_tc_min_macs;
}

template <bool TA, bool TB>
cudaError_t dispatch(int M, int N, int K, const float* A, int lda, const float* B, int ldb, float* C, int ldc,
                     float beta, cudaStream_t s) {
    const bool vec = lda % 4 == 0 && ldb % 4 == 0 && ((uintptr_t)A & 15) == 0 && ((uintptr_t)B & 15) == 0;
    const int64_t tmin = tc_min_macs();
    if (vec && tmin >= 0 && M >= 64 && N >= 64 && K >= 64 && (int64_t)M * N * K >= tmin)
        return tc::launch<TA, TB>(M, N, K, A, lda, B, ldb, C, ldc, beta, s);
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
