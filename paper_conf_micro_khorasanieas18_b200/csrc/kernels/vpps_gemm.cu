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

// ---- tensor-core tiles: tcgen05.mma kind::tf32 with a 3xTF32 split (FP32 accuracy) -------------------------
// Large products (the C5-sized level products and per-matrix gradient GEMMs: a level batches enough
// same-parameter nodes to form a real dense GEMM, north_star) run on the 5th-gen tensor cores.
// D[128 x 128] per CTA accumulates in TMEM (128 columns).  K runs in chunks of 32 through two shared-memory
// stages; every thread stages its share of a chunk through registers — 16-byte global loads along the
// operand's contiguous dimension, split v = hi + lo (hi = v truncated to TF32, lo = v - hi exact in FP32) and
// stored in the K-major SWIZZLE_NONE canonical layout (core matrix 8 rows x 16 B, SBO 128 B between 8-row
// groups; LBO = 2064 B between 4-k slices — 16 B of padding make both the 16-byte stores of K-contiguous
// operands and the 4-byte transposing stores of M/N-contiguous ones bank-conflict free).  One thread issues
// D += A·B + A·B_lo + A_lo·B per k-step of 8 (the dropped A_lo·B_lo is ~2^-22 relative) and commits to the
// stage's mbarrier; the loads of chunk c + 1 are in flight while chunk c is converted and multiplied.
namespace tc {
constexpr int BM = 128, BN = 128, BKC = 32, NT = 256;
constexpr uint32_t LBO = (BM / 8) * 128 + 16;                 // bytes between 4-k slices (padded)
constexpr int OP_F = (BKC / 4) * (LBO / 4);                    // floats of one operand copy (hi or lo)
constexpr int STAGE_F = 4 * OP_F;                              // A hi, A lo, B hi, B lo
constexpr size_t SMEM = (size_t)2 * STAGE_F * sizeof(float) + 128;
static_assert(BM == BN, "one staging geometry for both operands");

__device__ __forceinline__ uint64_t desc(uint32_t saddr) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((LBO >> 4) & 0x3FFF) << 16) |
           ((uint64_t)(128 >> 4) << 32) | ((uint64_t)1 << 46);
}
constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
__device__ __forceinline__ void mma(uint32_t d, uint64_t a, uint64_t b, int acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n"
                 ::"r"(d), "l"(a), "l"(b), "r"(IDESC), "r"(acc));
}
__device__ __forceinline__ void mbar_wait(uint32_t mbar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
                     : "=r"(ok) : "r"(mbar), "r"(parity) : "memory");
}
__device__ __forceinline__ float tf32_hi(float v) { return __uint_as_float(__float_as_uint(v) & 0xFFFFE000u); }

// one operand's share of a chunk: 4 x 16-byte pieces per thread.  KC (contiguous along k): piece g = row
// g / 8, k4 = g % 8; otherwise (contiguous along rows) lane = k, piece = 4 consecutive rows 4 (g / 32)
template <bool KC>
__device__ __forceinline__ void load_chunk(const float* __restrict__ X, int ld, int r0, int rmax, int k0, int kmax,
                                           float4 (&v)[4]) {
#pragma unroll
    for (int p = 0; p < 4; ++p) {
        const int g = threadIdx.x + NT * p;
        const int r = KC ? g / 8 : 4 * (g / 32), k = KC ? 4 * (g % 8) : g % 32;
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
// element (r, k) of a stage copy: float offset (k / 4) (LBO / 4) + (r / 8) 32 + (r % 8) 4 + k % 4
template <bool KC>
__device__ __forceinline__ void store_chunk(float* hi, float* lo, const float4 (&v)[4]) {
#pragma unroll
    for (int p = 0; p < 4; ++p) {
        const int g = threadIdx.x + NT * p;
        if (KC) {
            const int r = g / 8, k4 = g % 8;
            const int o = k4 * (LBO / 4) + (r >> 3) * 32 + (r & 7) * 4;
            const float4 h = make_float4(tf32_hi(v[p].x), tf32_hi(v[p].y), tf32_hi(v[p].z), tf32_hi(v[p].w));
            *reinterpret_cast<float4*>(hi + o) = h;
            *reinterpret_cast<float4*>(lo + o) = make_float4(v[p].x - h.x, v[p].y - h.y, v[p].z - h.z, v[p].w - h.w);
        } else {
            const int r0 = 4 * (g / 32), k = g % 32;
            const float e[4] = {v[p].x, v[p].y, v[p].z, v[p].w};
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                const int r = r0 + q;
                const int o = (k >> 2) * (LBO / 4) + (r >> 3) * 32 + (r & 7) * 4 + (k & 3);
                const float h = tf32_hi(e[q]);
                hi[o] = h;
                lo[o] = e[q] - h;
            }
        }
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
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int m0 = blockIdx.y * BM, n0 = blockIdx.x * BN;
    const int kb = blockIdx.z * k_split, ke = min(K, kb + k_split);
    const int nch = (ke - kb + BKC - 1) / BKC;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base)), "r"(BN));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 32) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar[0])));
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar[1])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    float4 ra[4], rb[4];
    load_chunk<!TA>(A, lda, m0, M, kb, ke, ra);
    load_chunk<TB>(B, ldb, n0, N, kb, ke, rb);
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = tmem_base;
    uint32_t phases = 0u;                          // bit st: parity of stage st's next completion
    for (int c = 0; c < nch; ++c) {
        const int st = c & 1;
        float* Ah = sm + st * STAGE_F;
        float* Al = Ah + OP_F;
        float* Bh = Al + OP_F;
        float* Bl = Bh + OP_F;
        if (c >= 2) { mbar_wait(smem_u32(&mbar[st]), (phases >> st) & 1u); phases ^= 1u << st; }   // chunk c - 2 read it
        store_chunk<!TA>(Ah, Al, ra);
        store_chunk<TB>(Bh, Bl, rb);
        if (c + 1 < nch) {                        // next chunk's loads in flight during this chunk's MMAs
            load_chunk<!TA>(A, lda, m0, M, kb + (c + 1) * BKC, ke, ra);
            load_chunk<TB>(B, ldb, n0, N, kb + (c + 1) * BKC, ke, rb);
        }
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic smem writes -> tensor core
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncthreads();
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        if (tid == 0) {
            const uint32_t a0 = smem_u32(Ah), al0 = smem_u32(Al), b0 = smem_u32(Bh), bl0 = smem_u32(Bl);
#pragma unroll
            for (int s = 0; s < BKC / 8; ++s) {
                const uint32_t o = 2 * s * LBO;
                mma(tmem, desc(a0 + o), desc(b0 + o), c > 0 || s > 0);
                mma(tmem, desc(a0 + o), desc(bl0 + o), 1);
                mma(tmem, desc(al0 + o), desc(b0 + o), 1);
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                         ::"r"(smem_u32(&mbar[st])) : "memory");
        }
    }
    // the last commit covers every earlier MMA
    if (nch > 0) {
        const int st = (nch - 1) & 1;
        mbar_wait(smem_u32(&mbar[st]), (phases >> st) & 1u);
    }
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    // epilogue: warp w reads TMEM lanes 32 (w & 3) .. (rows), columns 64 (w >> 2) .. +63
    const int row = m0 + 32 * (warp & 3) + lane, cb = 64 * (warp >> 2);
    const bool split = gridDim.z > 1;
    const bool vec = (ldc & 3) == 0 && ((reinterpret_cast<uintptr_t>(C) & 15) == 0);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        uint32_t r[16];
        const uint32_t ta = tmem + ((uint32_t)(32 * (warp & 3)) << 16) + cb + 16 * q;
        asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                     : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                       "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                     : "r"(ta));
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
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
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(BN));
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
