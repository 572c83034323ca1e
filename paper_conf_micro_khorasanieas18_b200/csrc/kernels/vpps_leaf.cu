// The leaf level of the binary Tree-LSTM as a dense GEMM with the leaf cell fused into its epilogue
// (cluster path).
//
// Every leaf of a batch uses the same matrix W_iou on its word vector (words enter the
// Tree-LSTM at the leaves), so level 0 is one dense GEMM — the case where north_star allows a GEMM
// instead of per-node matrix-vector products.  The recurrent matrices (U_iou, U_fl, U_fr) stay
// register-resident in vpps_cl.
//
//   vpps_leaf_fwd: a = W_iou x_l + b_iou; i, o = σ, u = tanh; c = i u; h = o tanh c  -> leaf record [h c i o u]
//
// Tile: 64 leaves x 16 hidden units x 3 gates (i, o, u of the same units, so the cell can run in the
// epilogue), 256 threads, one CTA per SM: the TGT batch (~450 leaves) is one wave of 128 CTAs and the
// remaining CTAs only clear.  The K range is issued as 4 cp.async groups of 64 columns up front and
// consumed as the groups land.  Four K slices of 64
// threads take alternating 4-column steps; thread (slice, lg, up) owns leaves lg + 8a (a < 8) x units
// 2up, 2up+1 x 3 gates (48 accumulators): per 4-column step 8 + 6 LDS.128 (conflict-free: row stride =
// 4 mod 32 words) feed 192 FFMA.  The slices are summed through shared memory and one (leaf, unit) pair
// per thread runs the cell.  (A 4 x 3 thread tile was shared-memory-issue bound: mio_throttle and short
// scoreboard stalls, FMA pipe 30 %, 13 us per TGT pass, profiles/r03 ncu.)
// The input-table gradient dX = W_iouᵀ g_leaf is a job of the gradient GEMM (vpps_dw_gemm, vpps_cluster.cu).
// Requires E in {128, 256} (the tensor-core variant: E == 256) and H % 16 == 0.
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <cuda.h>
#include <cudaTypedefs.h>
#include "vpps_kernel.cuh"
#include "dev_common.cuh"

namespace vpps {
namespace dev {
namespace leaf {

constexpr int LM = 64;          // leaves per tile
constexpr int LU = 16;          // hidden units per tile (x 3 gates = 48 W_iou rows)
constexpr int NT = 256;         // 4 K slices (alternating 4-column steps) x 64 threads
constexpr int NTC = 128;        // + 4 warps that only clear (warp-specialised: the GEMM never waits for them)
constexpr int KMAX = 256;       // largest E (the tensor-core variant: E == KMAX)
constexpr int KST = 64;         // K columns per cp.async group (E / KST groups)
// row stride in floats E + 4 (= 4 mod 32: conflict-free 16-byte column reads)
template <int E>
constexpr size_t smem_of() { return (size_t)(LM + 3 * LU) * (E + 4) * sizeof(float); }

// Per-pass clearing folded into the leaf kernel (it runs first in the pass): up to 4 float ranges
// (multiples of 4 floats) are zeroed by a grid-stride loop, and the device pass counter is advanced.
__device__ uint64_t g_leaf_prof[1024 * 8];   // measurement only (VPPS_LEAF_PROF): per-CTA phase stamps
__device__ int g_leaf_prof_on;
static int h_leaf_prof_on = 0;   // host copy: selects the trace-enabled instantiation (PROF = true)

// barrier of the NT GEMM threads only (the clearing warps never join it)
__device__ __forceinline__ void gemm_sync() { asm volatile("bar.sync 1, %0;" ::"n"(NT) : "memory"); }

struct PassClear {
    float* ptr[4];
    int64_t n[4];
    uint32_t* epoch;     // dataflow pass counter (tags of this pass), or nullptr
    const char* pf;      // bytes to pull into L2 for the next kernel (the dataflow kernel's weights), or nullptr
    int64_t pf_bytes;
};

template <int E, bool PROF>
__global__ void __launch_bounds__(NT + NTC, 1) vpps_leaf_fwd(const float* __restrict__ W, const float* __restrict__ b,
                                                       const float* __restrict__ inputs, float* pool,
                                                       const uint32_t* __restrict__ leaves, int n_leaf, int H,
                                                       const PassClear pc) {
    static_assert(E == 128 || E == 256, "leaf GEMM: E in {128, 256}");
    constexpr int NSTG = E / KST, KS = E + 4;
    extern __shared__ __align__(16) float lsm[];
    __shared__ uint32_t lrec[LM];
    float* As = lsm;                 // [64 leaves][KS]: x rows
    float* Bs = lsm + LM * KS;       // [48 rows][KS]: W_iou rows g*H + j0 + uu, row index g*16 + uu
    const int tid = threadIdx.x;
    // the dataflow kernel may be scheduled as SMs free up (it waits for this grid with griddepcontrol.wait
    // before reading anything written here)
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    // production instantiation: no trace (the flag load and the stamps fold away)
    const bool pf = PROF && tid == 0 && blockIdx.x < 1024 && g_leaf_prof_on;
    uint64_t* pst = g_leaf_prof + blockIdx.x * 8;
    if (pf) pst[0] = gtimer();
    if (pc.epoch && blockIdx.x == 0 && tid == 0) {
        uint32_t e = *pc.epoch + 1;
        *pc.epoch = e ? e : 1u;                                   // 0 marks never-written slots
    }
    const int tiles_u = H / LU;
    const int l0 = (blockIdx.x / tiles_u) * LM, j0 = (blockIdx.x % tiles_u) * LU;
    const bool work = l0 < n_leaf;
    if (tid >= NT) {   // clearing warps: per-pass clearing while the GEMM warps stage and compute
        const int64_t stride = (int64_t)gridDim.x * NTC;
        for (int r = 0; r < 4; ++r) {
            float4* p = reinterpret_cast<float4*>(pc.ptr[r]);
            const int64_t n4 = pc.ptr[r] ? pc.n[r] / 4 : 0;
            for (int64_t i = (int64_t)blockIdx.x * NTC + (tid - NT); i < n4; i += stride) p[i] = make_float4(0.f, 0.f, 0.f, 0.f);
        }
        // pull the dataflow kernel's recurrent weights into L2 meanwhile: its prologue (registers of every
        // CTA, after this grid's CTAs have left the SMs) then reads L2 instead of DRAM
        for (int64_t i = (int64_t)blockIdx.x * NTC + (tid - NT); i < pc.pf_bytes / 128; i += stride)
            asm volatile("prefetch.global.L2 [%0];" ::"l"(pc.pf + i * 128));
        if (PROF && tid == NT && blockIdx.x < 1024 && g_leaf_prof_on) g_leaf_prof[blockIdx.x * 8 + 6] = gtimer();
        return;
    }
    if (work) {
        // staging: thread tid issues the 16-byte pieces (row tid/16 + 16p, column piece tid%16) of every
        // K group, W rows (48) and x rows (64) alike; tokens first (one round trip)
        constexpr int PPR = KST / 4;                 // pieces per row per group
        const int pc_ = tid % PPR, r0 = tid / PPR;   // r0 < 16
        uint32_t tok[LM / 16];
#pragma unroll
        for (int p = 0; p < LM / 16; ++p) {
            const int l = l0 + r0 + 16 * p;
            tok[p] = l < n_leaf ? __ldg(leaves + 2 * l + 1) : 0xFFFFFFFFu;
        }
        if (tid < LM) lrec[tid] = l0 + tid < n_leaf ? __ldg(leaves + 2 * (l0 + tid)) : 0u;
#pragma unroll
        for (int s = 0; s < NSTG; ++s) {
            const int c = s * KST + 4 * pc_;
#pragma unroll
            for (int p = 0; p < 3; ++p)              // W row r0 + 16p = gate p, unit r0
                cp_async16(Bs + (r0 + 16 * p) * KS + c, W + (int64_t)(p * H + j0 + r0) * E + c, 16u);
#pragma unroll
            for (int p = 0; p < LM / 16; ++p) {
                const bool ok = tok[p] != 0xFFFFFFFFu;
                cp_async16(As + (r0 + 16 * p) * KS + c, ok ? inputs + (int64_t)tok[p] * E + c : W, ok ? 16u : 0u);
            }
            asm volatile("cp.async.commit_group;" ::: "memory");
        }
    }
    if (pf) pst[1] = gtimer();
    if (!work) return;                                             // clearing-only CTA
    const int ks = tid >> 6, t64 = tid & 63, lg = t64 & 7, up = t64 >> 3;   // K slice, leaves lg + 8a, units 2up + c
    float acc[8][6];
#pragma unroll
    for (int a = 0; a < 8; ++a)
#pragma unroll
        for (int q = 0; q < 6; ++q) acc[a][q] = 0.f;
    const float* ap = As + lg * KS;
    const float* bw = Bs + 2 * up * KS;
    auto stage = [&](int s) {
#pragma unroll 2
        for (int k = s * KST + 4 * ks; k < (s + 1) * KST; k += 16) {
            float4 w[6];
#pragma unroll
            for (int g = 0; g < 3; ++g)
#pragma unroll
                for (int c = 0; c < 2; ++c) w[g * 2 + c] = *reinterpret_cast<const float4*>(bw + (g * LU + c) * KS + k);
#pragma unroll
            for (int a = 0; a < 8; ++a) {
                const float4 x = *reinterpret_cast<const float4*>(ap + 8 * a * KS + k);
#pragma unroll
                for (int q = 0; q < 6; ++q)
                    acc[a][q] = fmaf(x.w, w[q].w, fmaf(x.z, w[q].z, fmaf(x.y, w[q].y, fmaf(x.x, w[q].x, acc[a][q]))));
            }
        }
    };
    if constexpr (NSTG == 4) {
        asm volatile("cp.async.wait_group 3;" ::: "memory");
        gemm_sync();
        if (pf) pst[2] = gtimer();
        stage(0);
        asm volatile("cp.async.wait_group 2;" ::: "memory");
        gemm_sync();
        stage(1);
    } else {
        static_assert(NSTG == 2, "E / KST cp.async groups: 2 or 4");
    }
    asm volatile("cp.async.wait_group 1;" ::: "memory");
    gemm_sync();
    if (NSTG == 2 && pf) pst[2] = gtimer();
    stage(NSTG - 2);
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    gemm_sync();
    if (pf) pst[3] = gtimer();
    stage(NSTG - 1);
    if (pf) pst[4] = gtimer();
    // sum the K slices through shared memory (the staging is dead): red[slice][t64][49]
    constexpr int RS = 49;
    gemm_sync();
    float* red = lsm;
#pragma unroll
    for (int a = 0; a < 8; ++a)
#pragma unroll
        for (int q = 0; q < 6; ++q) red[(ks * 64 + t64) * RS + a * 6 + q] = acc[a][q];
    gemm_sync();
    // cell: pair (leaf l, unit uu) per thread pass, consecutive threads on consecutive units (coalesced)
#pragma unroll
    for (int pp = 0; pp < LM * LU / NT; ++pp) {
        const int pr = tid + NT * pp, uu = pr % LU, li = pr / LU;
        if (l0 + li >= n_leaf) break;
        const int src = (li & 7) + 8 * (uu >> 1), col = (li >> 3) * 6 + (uu & 1);
        float pre[3];
#pragma unroll
        for (int g = 0; g < 3; ++g) {
            float v = 0.f;
#pragma unroll
            for (int q = 0; q < 4; ++q) v += red[(q * 64 + src) * RS + col + 2 * g];
            pre[g] = v;
        }
        const int j = j0 + uu;
        float* r = pool + lrec[li];
        const float ig = fsigm(pre[0] + __ldg(b + j)), og = fsigm(pre[1] + __ldg(b + H + j));
        const float ug = ftanh(pre[2] + __ldg(b + 2 * H + j));
        const float cc = ig * ug;
        r[j] = og * ftanh(cc);
        r[H + j] = cc;
        r[2 * H + j] = ig;
        r[3 * H + j] = og;
        r[4 * H + j] = ug;
    }
    if (pf) pst[5] = gtimer();
}


// ---- tensor-core variant (opt-in, VPPS_LEAF_TC=1): the leaf GEMM as tcgen05.mma kind::tf32 with a 3xTF32 split ----
// D[128 leaves][48 rows] = Σ_k x[leaf][k] W_iou[row][k]: both operands are K-major as they lie in memory
// (embedding rows, W_iou rows), so each thread stages 16-byte k-pieces through registers, splitting
// v = hi + lo (hi = v truncated to TF32, lo = v - hi exact in FP32) into the SWIZZLE_NONE canonical layout
// (core matrix = 8 rows x 16 B; rows 16 B apart, SBO = 128 B between 8-row groups, LBO = (rows/8)*128 B
// between 4-k chunks; the layout tools/umma_test.cu pins).  D = A·B + A·B_lo + A_lo·B (the dropped
// A_lo·B_lo is ~2^-22 relative: FP32 accuracy, parity bar 1e-4) accumulates in TMEM (48 of 64 columns).
// K runs in 4 chunks of 64 through two smem buffers: the MMAs of chunk c (issued by one thread, completion
// on an mbarrier) overlap the global loads and conversion of chunk c + 1.  Epilogue: tcgen05.ld of the
// i, o, u columns of 8 units per thread (warp w: TMEM lanes 32(w&3).., units 8(w>>2)..), cell, 16-byte
// record stores.  Tile count for the TGT batch (~450 leaves): 4 x 16 = 64 CTAs; the CTAs behind the tiles
// (the leftover SMs, at least 32) do the per-pass clearing.
constexpr int TL = 128;                 // leaves per tile (UMMA M)
constexpr int TR = 3 * LU;              // W_iou rows per tile (UMMA N = 48)
constexpr int KC = 64;                  // K per chunk
constexpr int NCH = KMAX / KC;
static_assert(NCH == 4, "chunk / mbarrier phase sequence below assumes 4 chunks");
constexpr int A_F = TL * KC, B_F = TR * KC;          // floats per hi (or lo) copy
constexpr int BUF_F = 2 * A_F + 2 * B_F;
constexpr size_t TC_SMEM = (size_t)2 * BUF_F * sizeof(float);
constexpr uint32_t LBO_A = (TL / 8) * 128, LBO_B = (TR / 8) * 128;   // bytes between 4-k chunks

__device__ __forceinline__ uint64_t lf_desc(uint32_t saddr, uint32_t lbo) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)(128 >> 4) << 32) | ((uint64_t)1 << 46);
}
constexpr uint32_t lf_idesc(int m, int n) {      // F32 accumulate, TF32 A/B, both K-major
    return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(m >> 4) << 24);
}
__device__ __forceinline__ void lf_mma(uint32_t d, uint64_t a, uint64_t b, int acc) {
    constexpr uint32_t idesc = lf_idesc(TL, TR);
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n"
                 ::"r"(d), "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void lf_wait(uint32_t mbar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
                     : "=r"(ok) : "r"(mbar), "r"(parity) : "memory");
}
__device__ __forceinline__ void split_store(float* hi, float* lo, uint32_t off, const float4 v) {
    const float4 h = make_float4(__uint_as_float(__float_as_uint(v.x) & 0xFFFFE000u), __uint_as_float(__float_as_uint(v.y) & 0xFFFFE000u),
                                 __uint_as_float(__float_as_uint(v.z) & 0xFFFFE000u), __uint_as_float(__float_as_uint(v.w) & 0xFFFFE000u));
    *reinterpret_cast<float4*>(hi + off) = h;
    *reinterpret_cast<float4*>(lo + off) = make_float4(v.x - h.x, v.y - h.y, v.z - h.z, v.w - h.w);
}
__device__ __forceinline__ void mbar_wait_parity(uint32_t mbar, uint32_t parity) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
                     : "=r"(ok) : "r"(mbar), "r"(parity) : "memory");
}
__device__ __forceinline__ void tcl_ld16(uint32_t ta, uint32_t (&r)[16]) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                 : "r"(ta));
}
#define LF_LD8(r, addr)                                                                                        \
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"                     \
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]) \
                 : "r"(addr))

__global__ void __launch_bounds__(NT, 1) vpps_leaf_fwd_tc(const float* __restrict__ W, const float* __restrict__ b,
                                                        const float* __restrict__ inputs, float* pool,
                                                        const uint32_t* __restrict__ leaves, int n_leaf, int H,
                                                        int tiles, const PassClear pc) {
    extern __shared__ __align__(128) float tsm[];
    __shared__ uint32_t tmem_base;
    __shared__ __align__(8) uint64_t mbar[2];
    __shared__ float bias_s[3 * LU];
    const int tid = threadIdx.x;
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const bool pf = g_leaf_prof_on && tid == 0 && blockIdx.x < 1024;
    uint64_t* pst = g_leaf_prof + blockIdx.x * 8;
    if (pf) pst[0] = gtimer();
    if ((int)blockIdx.x >= tiles) {
        // clearing CTAs (the GEMM tiles never wait for the per-pass clearing) and the pass counter
        const int cb = blockIdx.x - tiles, ncb = gridDim.x - tiles;
        if (pc.epoch && cb == 0 && tid == 0) {
            uint32_t e = *pc.epoch + 1;
            *pc.epoch = e ? e : 1u;                               // 0 marks never-written slots
        }
        const int64_t stride = (int64_t)ncb * NT;
        for (int r = 0; r < 4; ++r) {
            float4* p = reinterpret_cast<float4*>(pc.ptr[r]);
            const int64_t n4 = pc.ptr[r] ? pc.n[r] / 4 : 0;
            for (int64_t i = (int64_t)cb * NT + tid; i < n4; i += stride) p[i] = make_float4(0.f, 0.f, 0.f, 0.f);
        }
        if (pf) pst[6] = gtimer();
        return;
    }
    const int tiles_u = H / LU;
    const int l0 = (blockIdx.x / tiles_u) * TL, j0 = (blockIdx.x % tiles_u) * LU;
    const int warp = tid >> 5, lane = tid & 31;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base)), "r"(64));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (tid == 32) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar[0])));
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar[1])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    if (tid >= 64 && tid < 64 + 3 * LU) {                          // b_iou of the tile's units
        const int k = tid - 64;
        bias_s[k] = __ldg(b + (k / LU) * H + j0 + k % LU);
    }
    // epilogue leaf of this thread (TMEM lane 32 (w & 3) + lane): its record offset, fetched early
    const int eq = warp & 3, eh = warp >> 2, eli = 32 * eq + lane;
    const uint32_t erec = l0 + eli < n_leaf ? __ldg(leaves + 2 * (l0 + eli)) : 0u;
    // staging: A row (leaf l0 + (tid & 127)), pieces k4 = ak0 + 2p (p < 8); B pieces e = tid + 256p:
    // row e % 48, k4 = e / 48.  Two chunks of registers in flight.
    const int ar = tid & (TL - 1), ak0 = tid >> 7;
    const uint32_t tok = l0 + ar < n_leaf ? __ldg(leaves + 2 * (l0 + ar) + 1) : 0xFFFFFFFFu;
    const float* arow = tok != 0xFFFFFFFFu ? inputs + (int64_t)tok * KMAX : nullptr;
    const float* brow[3];
    int bk4[3];
#pragma unroll
    for (int p = 0; p < 3; ++p) {
        const int e = tid + NT * p, r = e % TR;
        bk4[p] = e / TR;
        brow[p] = W + (int64_t)((r / LU) * H + j0 + r % LU) * KMAX;
    }
    float4 ra[2][8], rb[2][3];
    auto load = [&](int c, int set) {
#pragma unroll
        for (int p = 0; p < 8; ++p)
            ra[set][p] = arow ? __ldg(reinterpret_cast<const float4*>(arow + c * KC + 4 * (ak0 + 2 * p))) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
        for (int p = 0; p < 3; ++p) rb[set][p] = __ldg(reinterpret_cast<const float4*>(brow[p] + c * KC + 4 * bk4[p]));
    };
    load(0, 0);
    load(1, 1);
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = tmem_base;
    if (pf) pst[1] = gtimer();
#pragma unroll
    for (int c = 0; c < NCH; ++c) {
        const int set = c & 1;
        float* buf = tsm + set * BUF_F;
        float* Ah = buf;
        float* Al = Ah + A_F;
        float* Bh = Al + A_F;
        float* Bl = Bh + B_F;
        if (c >= 2) lf_wait(smem_u32(&mbar[set]), 0);             // the MMAs of chunk c - 2 have read the buffer
#pragma unroll
        for (int p = 0; p < 8; ++p) {
            const int k4 = ak0 + 2 * p;
            split_store(Ah, Al, (uint32_t)((ar >> 3) * 32 + (ar & 7) * 4 + k4 * (LBO_A / 4)), ra[set][p]);
        }
#pragma unroll
        for (int p = 0; p < 3; ++p) {
            const int e = tid + NT * p, r = e % TR;
            split_store(Bh, Bl, (uint32_t)((r >> 3) * 32 + (r & 7) * 4 + bk4[p] * (LBO_B / 4)), rb[set][p]);
        }
        if (c + 2 < NCH) load(c + 2, set);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic smem writes -> tensor core
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncthreads();
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        if (c == 0 && pf) pst[2] = gtimer();
        if (tid == 0) {
            const uint32_t a0 = smem_u32(Ah), al0 = smem_u32(Al), b0 = smem_u32(Bh), bl0 = smem_u32(Bl);
#pragma unroll
            for (int s = 0; s < KC / 8; ++s) {
                const uint64_t a = lf_desc(a0 + 2 * s * LBO_A, LBO_A), al = lf_desc(al0 + 2 * s * LBO_A, LBO_A);
                const uint64_t bb = lf_desc(b0 + 2 * s * LBO_B, LBO_B), bl = lf_desc(bl0 + 2 * s * LBO_B, LBO_B);
                lf_mma(tmem, a, bb, c > 0 || s > 0);
                lf_mma(tmem, a, bl, 1);
                lf_mma(tmem, al, bb, 1);
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                         ::"r"(smem_u32(&mbar[set])) : "memory");
        }
    }
    if (pf) pst[3] = gtimer();
    lf_wait(smem_u32(&mbar[1]), 1);                                // chunk 3 (and every earlier MMA) done
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (pf) pst[4] = gtimer();
    // epilogue: warp w reads TMEM lanes 32 (w & 3) .. +31 (leaves), the i / o / u columns of units 8 (w >> 2) .. +7
    {
        const uint32_t ta = tmem + ((uint32_t)(32 * eq) << 16) + 8 * eh;
        uint32_t gi[8], go[8], gu[8];
        LF_LD8(gi, ta);
        LF_LD8(go, ta + LU);
        LF_LD8(gu, ta + 2 * LU);
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        if (l0 + eli < n_leaf) {
            const int jb = j0 + 8 * eh;
            float* r = pool + erec;
            float hv[8], cv[8], iv[8], ov[8], uv[8];
#pragma unroll
            for (int t = 0; t < 8; ++t) {
                const int u = 8 * eh + t;
                const float ig = fsigm(__uint_as_float(gi[t]) + bias_s[u]);
                const float og = fsigm(__uint_as_float(go[t]) + bias_s[LU + u]);
                const float ug = ftanh(__uint_as_float(gu[t]) + bias_s[2 * LU + u]);
                const float cc = ig * ug;
                hv[t] = og * ftanh(cc); cv[t] = cc; iv[t] = ig; ov[t] = og; uv[t] = ug;
            }
#pragma unroll
            for (int t = 0; t < 8; t += 4) {
                *reinterpret_cast<float4*>(r + jb + t) = make_float4(hv[t], hv[t + 1], hv[t + 2], hv[t + 3]);
                *reinterpret_cast<float4*>(r + H + jb + t) = make_float4(cv[t], cv[t + 1], cv[t + 2], cv[t + 3]);
                *reinterpret_cast<float4*>(r + 2 * H + jb + t) = make_float4(iv[t], iv[t + 1], iv[t + 2], iv[t + 3]);
                *reinterpret_cast<float4*>(r + 3 * H + jb + t) = make_float4(ov[t], ov[t + 1], ov[t + 2], ov[t + 3]);
                *reinterpret_cast<float4*>(r + 4 * H + jb + t) = make_float4(uv[t], uv[t + 1], uv[t + 2], uv[t + 3]);
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(64));
    if (pf) pst[5] = gtimer();
}


// ---- TMA-fed tensor-core variant (opt-in, VPPS_LEAF_TMA=1): vpps_leaf_fwd_tma ----
// D[128 leaves][48 rows] = Σ_k x[tok_l][k] W_iou[row][k] as tcgen05.mma kind::tf32 with both operands fed by
// the Tensor Memory Accelerator: the leaf rows gathered by token (cp.async.bulk.tensor.2d ... tile::gather4,
// 4 rows per copy) and the 3 x 16 W_iou rows of the tile's units as 2D tiles, K-major in the SWIZZLE_128B
// layout (8-row x 128-byte atoms; the UMMA descriptor advances 32 B per k-step of 8).  The tensor core
// reads an FP32 operand as TF32 by truncation (tools/tma_probe.cu pins it: raw TF32 2.4e-4, 3xTF32 with
// lo = v - trunc(v) 7.6e-7 relative), so the raw tiles are the hi halves and six converter warps only write
// the lo halves (elementwise, same swizzled offsets): D = A·B + A·B_lo + A_lo·B, FP32 accuracy.
// Warp roles: warp 0 issues the TMA copies of every 32-column K chunk at once (8 raw chunks of 22 KB),
// warps 2-7 write the lo halves into a 2-stage ring, warp 1 issues the MMAs (12 per chunk) and frees a lo
// stage by tcgen05.commit; warps 4-7 then read the accumulator (TMEM lane = leaf) and run the leaf cell.
// CTAs behind the tiles do the per-pass clearing and pull vpps_df's recurrent weights into L2.
// Parity-green but measured slower than the FFMA tiles (TGT step 133 -> 145 us; leaf phase ~20 vs ~9 us):
// the 32 gather4 copies per K chunk (4 rows x 128 B each, the widest box SWIZZLE_128B allows) arrive one
// chunk per ~1.5 us, while the MMAs of a chunk take ~0.3 us (tools/tma_probe.cu: M = 128, N = 48 kind::tf32
// 50 cycles per MMA, N = 128 65 cycles = the TF32 peak).
namespace tma {
constexpr int ML = 128, NR = 48, KCT = 32;
constexpr int NRAW = 8, NLO = 2;                                     // raw chunks (all of K <= 256) / lo stages
constexpr int A_BYTES = ML * KCT * 4, B_BYTES = NR * KCT * 4;          // one raw chunk (16 KB, 6 KB)
constexpr int STAGE_BYTES = A_BYTES + B_BYTES;                       // A | B of one chunk (raw or lo)
constexpr size_t SMEM = (size_t)(NRAW + NLO) * STAGE_BYTES + 1024;
constexpr int NCONV = 192;                                           // converter threads (warps 2-7)
constexpr uint32_t IDESC = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(NR >> 3) << 17) | ((uint32_t)(ML >> 4) << 24);

__device__ __forceinline__ uint64_t desc_sw128(uint32_t saddr) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
           ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__device__ __forceinline__ void mma(uint32_t d, uint64_t a, uint64_t b, int acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n"
                 ::"r"(d), "l"(a), "l"(b), "r"(IDESC), "r"(acc));
}
__device__ __forceinline__ void arrive(uint32_t mbar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(mbar) : "memory");
}
}  // namespace tma

__global__ void __launch_bounds__(256, 1) vpps_leaf_fwd_tma(const __grid_constant__ CUtensorMap tmX,
                                                          const __grid_constant__ CUtensorMap tmW,
                                                          const float* __restrict__ b, float* pool,
                                                          const uint32_t* __restrict__ leaves, int n_leaf, int H, int E,
                                                          int tiles, const PassClear pc) {
    using namespace tma;
    extern __shared__ __align__(1024) uint8_t msm[];
    uint8_t* sm = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(msm) + 1023) & ~uintptr_t(1023));
    __shared__ uint32_t tmem_base;
    __shared__ __align__(8) uint64_t full[NRAW], lo_full[NLO], lo_empty[NLO], done;
    __shared__ float bias_s[3 * LU];
    __shared__ int tok_s[ML];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const bool pfon = g_leaf_prof_on && blockIdx.x < 1024;           // measurement only (tools/leaf_prof.py)
    const bool pf = pfon && tid == 0;
    uint64_t* pst = g_leaf_prof + blockIdx.x * 8;
    if (pf) pst[0] = gtimer();
    if ((int)blockIdx.x >= tiles) {
        // clearing CTAs: per-pass clearing, the pass counter, and vpps_df's recurrent weights into L2
        const int cb = blockIdx.x - tiles, ncb = gridDim.x - tiles;
        if (pc.epoch && cb == 0 && tid == 0) {
            uint32_t e = *pc.epoch + 1;
            *pc.epoch = e ? e : 1u;                               // 0 marks never-written slots
        }
        const int64_t stride = (int64_t)ncb * 256;
        for (int r = 0; r < 4; ++r) {
            float4* p = reinterpret_cast<float4*>(pc.ptr[r]);
            const int64_t n4 = pc.ptr[r] ? pc.n[r] / 4 : 0;
            for (int64_t i = (int64_t)cb * 256 + tid; i < n4; i += stride) p[i] = make_float4(0.f, 0.f, 0.f, 0.f);
        }
        for (int64_t i = (int64_t)cb * 256 + tid; i < pc.pf_bytes / 128; i += stride)
            asm volatile("prefetch.global.L2 [%0];" ::"l"(pc.pf + i * 128));
        if (pf) pst[6] = gtimer();
        return;
    }
    const int tiles_u = H / LU;
    const int l0 = (blockIdx.x / tiles_u) * ML, j0 = (blockIdx.x % tiles_u) * LU;
    const int nch = E / KCT;
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tmem_base)), "r"(64));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
        // the tile's tokens (rows past n_leaf gather row 0; their results are dropped)
#pragma unroll
        for (int q = 0; q < ML / 32; ++q) {
            const int l = l0 + 32 * q + lane;
            tok_s[32 * q + lane] = l < n_leaf ? (int)__ldg(leaves + 2 * l + 1) : 0;
        }
    }
    if (tid == 32) {
        for (int st = 0; st < NRAW; ++st) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&full[st])));
        for (int st = 0; st < NLO; ++st) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&lo_full[st])), "r"(NCONV));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&lo_empty[st])));
        }
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&done)));
        asm volatile("fence.mbarrier_init.release.cluster;");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmX)) : "memory");
        asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmW)) : "memory");
    }
    if (tid >= 64 && tid < 64 + 3 * LU) {                          // b_iou of the tile's units
        const int k = tid - 64;
        bias_s[k] = __ldg(b + (k / LU) * H + j0 + k % LU);
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const uint32_t tmem = tmem_base;
    if (pf) pst[1] = gtimer();
    // raw chunk c at sm + c * STAGE_BYTES (every K chunk in flight at once), lo stage q after them
    auto raw_at = [&](int c) { return sm + c * STAGE_BYTES; };
    auto lo_at = [&](int q) { return sm + (NRAW + q) * STAGE_BYTES; };
    if (warp == 0) {
        if (lane == 0) {
            const uint64_t mx = reinterpret_cast<uint64_t>(&tmX), mw = reinterpret_cast<uint64_t>(&tmW);
            for (int c = 0; c < nch; ++c) {
                uint8_t* Ar = raw_at(c);
                uint8_t* Br = Ar + A_BYTES;
                const uint32_t fb = smem_u32(&full[c]);
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(fb), "r"(A_BYTES + B_BYTES) : "memory");
                for (int q = 0; q < ML / 4; ++q)
                    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
                                 " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                                 ::"r"(smem_u32(Ar + q * 512)), "l"(mx), "r"(c * KCT), "r"(tok_s[4 * q]), "r"(tok_s[4 * q + 1]),
                                   "r"(tok_s[4 * q + 2]), "r"(tok_s[4 * q + 3]), "r"(fb) : "memory");
                for (int g = 0; g < 3; ++g)
                    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
                                 " [%0], [%1, {%2, %3}], [%4];"
                                 ::"r"(smem_u32(Br + g * LU * 128)), "l"(mw), "r"(c * KCT), "r"(g * H + j0), "r"(fb) : "memory");
            }
        }
    } else if (warp == 1) {
        if (lane == 0) {
            for (int c = 0; c < nch; ++c) {
                const int q = c % NLO;
                mbar_wait_parity(smem_u32(&lo_full[q]), (c / NLO) & 1);
                asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                const uint32_t a = smem_u32(raw_at(c)), bb = a + A_BYTES, al = smem_u32(lo_at(q)), bl = al + A_BYTES;
#pragma unroll
                for (int k = 0; k < KCT / 8; ++k) {
                    const uint32_t o = 32 * k;
                    mma(tmem, desc_sw128(a + o), desc_sw128(bb + o), c > 0 || k > 0);
                    mma(tmem, desc_sw128(a + o), desc_sw128(bl + o), 1);
                    mma(tmem, desc_sw128(al + o), desc_sw128(bb + o), 1);
                }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                             ::"r"(smem_u32(&lo_empty[q])) : "memory");
            }
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];"
                         ::"r"(smem_u32(&done)) : "memory");
        }
    } else {
        // converters: lo = v - trunc_tf32(v) of the landed chunk, at the same (swizzled) offsets
        const int ct = tid - 64;
        for (int c = 0; c < nch; ++c) {
            const int q = c % NLO;
            mbar_wait_parity(smem_u32(&full[c]), 0);
            if (c >= NLO) mbar_wait_parity(smem_u32(&lo_empty[q]), ((c / NLO) - 1) & 1);   // chunk c - 2's MMAs
            if (pfon && ct == 0 && (c == 0 || c == nch - 1)) pst[c == 0 ? 2 : 3] = gtimer();
            const uint8_t* raw = raw_at(c);
            uint8_t* lo = lo_at(q);
            for (int i = ct; i < STAGE_BYTES / 16; i += NCONV) {
                const float4 v = *reinterpret_cast<const float4*>(raw + i * 16);
                const float4 h = make_float4(__uint_as_float(__float_as_uint(v.x) & 0xFFFFE000u), __uint_as_float(__float_as_uint(v.y) & 0xFFFFE000u),
                                             __uint_as_float(__float_as_uint(v.z) & 0xFFFFE000u), __uint_as_float(__float_as_uint(v.w) & 0xFFFFE000u));
                *reinterpret_cast<float4*>(lo + i * 16) = make_float4(v.x - h.x, v.y - h.y, v.z - h.z, v.w - h.w);
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic smem writes -> tensor core
            tma::arrive(smem_u32(&lo_full[q]));
        }
        if (warp >= 4) {
            // epilogue: warp w reads TMEM lanes 32 (w - 4) .. +31 = leaves, all 48 columns (i, o, u of 16 units)
            const int eli = 32 * (warp - 4) + lane;
            const uint32_t erec = l0 + eli < n_leaf ? __ldg(leaves + 2 * (l0 + eli)) : 0u;
            mbar_wait_parity(smem_u32(&done), 0);
            asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
            if (pfon && warp == 4 && lane == 0) pst[4] = gtimer();
            const uint32_t ta = tmem + ((uint32_t)(32 * (warp - 4)) << 16);
            uint32_t gi[16], go[16], gu[16];
            tcl_ld16(ta, gi);
            tcl_ld16(ta + LU, go);
            tcl_ld16(ta + 2 * LU, gu);
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
            if (l0 + eli < n_leaf) {
                float* r = pool + erec;
#pragma unroll
                for (int t = 0; t < LU; t += 4) {
                    float hv[4], cv[4], iv[4], ov[4], uv[4];
#pragma unroll
                    for (int q = 0; q < 4; ++q) {
                        const int u = t + q;
                        const float ig = fsigm(__uint_as_float(gi[u]) + bias_s[u]);
                        const float og = fsigm(__uint_as_float(go[u]) + bias_s[LU + u]);
                        const float ug = ftanh(__uint_as_float(gu[u]) + bias_s[2 * LU + u]);
                        const float cc = ig * ug;
                        hv[q] = og * ftanh(cc); cv[q] = cc; iv[q] = ig; ov[q] = og; uv[q] = ug;
                    }
                    *reinterpret_cast<float4*>(r + j0 + t) = make_float4(hv[0], hv[1], hv[2], hv[3]);
                    *reinterpret_cast<float4*>(r + H + j0 + t) = make_float4(cv[0], cv[1], cv[2], cv[3]);
                    *reinterpret_cast<float4*>(r + 2 * H + j0 + t) = make_float4(iv[0], iv[1], iv[2], iv[3]);
                    *reinterpret_cast<float4*>(r + 3 * H + j0 + t) = make_float4(ov[0], ov[1], ov[2], ov[3]);
                    *reinterpret_cast<float4*>(r + 4 * H + j0 + t) = make_float4(uv[0], uv[1], uv[2], uv[3]);
                }
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(64));
    if (pf) pst[5] = gtimer();
}

}  // namespace leaf
}  // namespace dev

extern "C" int vpps_leaf_prof(int on, uint64_t* out) {   // measurement tool hook (not in vpps.h)
    if (out) return (int)cudaMemcpyFromSymbol(out, dev::leaf::g_leaf_prof, sizeof(uint64_t) * 1024 * 8);
    dev::leaf::h_leaf_prof_on = on;
    return (int)cudaMemcpyToSymbol(dev::leaf::g_leaf_prof_on, &on, sizeof(int));
}

// 2D FP32 tensor map [rows][cols] (row stride cols * 4 bytes), box KCT columns x box_rows rows, SWIZZLE_128B;
// cuTensorMapEncodeTiled comes from the driver through the runtime's entry-point query (no libcuda link)
static bool encode_map(CUtensorMap* map, const float* base, int64_t rows, int64_t cols, int box_rows) {
    static PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
    static std::once_flag once;
    std::call_once(once, [] {
        void* fn = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            enc = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
    });
    if (!enc) return false;
    const cuuint64_t gd[2] = {(cuuint64_t)cols, (cuuint64_t)rows}, gs[1] = {(cuuint64_t)cols * 4};
    const cuuint32_t bx[2] = {(cuuint32_t)dev::leaf::tma::KCT, (cuuint32_t)box_rows}, es[2] = {1, 1};
    return enc(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), gd, gs, bx, es,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

void launch_leaf_fwd(const float* W, const float* b, const float* inputs, float* pool, const uint32_t* leaves,
                     int32_t n_leaf, int32_t H, int32_t E, float* const* zero_ptr, const int64_t* zero_n,
                     uint32_t* epoch, cudaStream_t s, const void* prefetch, int64_t prefetch_bytes, int64_t n_rows) {
    using namespace dev::leaf;
    if ((E != 128 && E != KMAX) || H % LU) return;   // (api.cu admits only built (H, E) variants)
    PassClear pc{};
    static const int exp_ = getenv("VPPS_LEAF_EXP") ? atoi(getenv("VPPS_LEAF_EXP")) : 0;   // measurement only
    // VPPS_LEAF_TC=1: the tensor-core variant (parity-green; measured slower than the FFMA tiles, 17.5 vs
    // 12.3 us per TGT pass: the register-transit staging of the hi / lo split and the first TMEM allocation
    // sit on its critical path)
    static const bool simt_env = !(getenv("VPPS_LEAF_TC") && atoi(getenv("VPPS_LEAF_TC")) != 0);
    const bool simt = simt_env || E != KMAX;
    for (int r = 0; r < 4; ++r) { pc.ptr[r] = zero_ptr ? zero_ptr[r] : nullptr; pc.n[r] = zero_ptr ? zero_n[r] : 0; }
    if (exp_ & 1) for (int r = 0; r < 4; ++r) if (r != 2) pc.n[r] = 0;     // no clearing (but the counters)
    if (exp_ & 2) n_leaf = 0;                                                // clearing only
    pc.epoch = epoch;
    pc.pf = static_cast<const char*>(prefetch);
    pc.pf_bytes = prefetch ? prefetch_bytes : 0;
    // VPPS_LEAF_TMA=1: the TMA-fed tensor-core tiles (parity-green, slower: see vpps_leaf_fwd_tma)
    static const bool tma_env = getenv("VPPS_LEAF_TMA") && atoi(getenv("VPPS_LEAF_TMA")) != 0;
    if (tma_env && n_rows > 0 && (E == 128 || E == 256) && H % LU == 0) {
        CUtensorMap mx, mw;
        if (encode_map(&mx, inputs, n_rows, E, 1) && encode_map(&mw, W, 3 * (int64_t)H, E, LU)) {
            // GEMM tiles first, then clearing CTAs: the SMs left over (at least 32 CTAs)
            const int tiles = ((n_leaf + tma::ML - 1) / tma::ML) * (H / LU);
            const int grid = tiles + std::max(148 - tiles, 32);
            vpps_leaf_fwd_tma<<<grid, 256, tma::SMEM, s>>>(mx, mw, b, pool, leaves, n_leaf, H, E, tiles, pc);
            return;
        }
    }
    if (simt) {
        const int tiles = std::max(((n_leaf + LM - 1) / LM) * (H / LU), 148);
        if (E == 128) {
            if (h_leaf_prof_on) vpps_leaf_fwd<128, true><<<tiles, NT + NTC, smem_of<128>(), s>>>(W, b, inputs, pool, leaves, n_leaf, H, pc);
            else vpps_leaf_fwd<128, false><<<tiles, NT + NTC, smem_of<128>(), s>>>(W, b, inputs, pool, leaves, n_leaf, H, pc);
        } else {
            if (h_leaf_prof_on) vpps_leaf_fwd<256, true><<<tiles, NT + NTC, smem_of<256>(), s>>>(W, b, inputs, pool, leaves, n_leaf, H, pc);
            else vpps_leaf_fwd<256, false><<<tiles, NT + NTC, smem_of<256>(), s>>>(W, b, inputs, pool, leaves, n_leaf, H, pc);
        }
    } else {
        // GEMM tiles first, then clearing CTAs: the SMs left over (at least 32 CTAs)
        const int tiles = ((n_leaf + TL - 1) / TL) * (H / LU);
        const int grid = tiles + std::max(148 - tiles, 32);
        vpps_leaf_fwd_tc<<<grid, NT, TC_SMEM, s>>>(W, b, inputs, pool, leaves, n_leaf, H, tiles, pc);
    }
}

// per-device launch attributes of the leaf kernels (vpps_define_model calls this after cudaSetDevice)
cudaError_t setup_leaf_attrs() {
    using namespace dev::leaf;
    cudaError_t e = cudaFuncSetAttribute(vpps_leaf_fwd<256, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_of<256>());
    if (e == cudaSuccess) e = cudaFuncSetAttribute(vpps_leaf_fwd<256, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_of<256>());
    if (e == cudaSuccess) e = cudaFuncSetAttribute(vpps_leaf_fwd<128, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_of<128>());
    if (e == cudaSuccess) e = cudaFuncSetAttribute(vpps_leaf_fwd<128, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_of<128>());
    if (e == cudaSuccess) e = cudaFuncSetAttribute(vpps_leaf_fwd_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)TC_SMEM);
    if (e == cudaSuccess) e = cudaFuncSetAttribute(vpps_leaf_fwd_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tma::SMEM);
    return e;
}

}  // namespace vpps
