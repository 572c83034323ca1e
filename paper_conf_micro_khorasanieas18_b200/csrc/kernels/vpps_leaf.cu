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
// Requires E == KMAX and H % 16 == 0 (the cluster / dataflow variants are H = E = 256).
#include <algorithm>
#include <cstdlib>
#include "vpps_kernel.cuh"
#include "dev_common.cuh"

namespace vpps {
namespace dev {
namespace leaf {

constexpr int LM = 64;          // leaves per tile
constexpr int LU = 16;          // hidden units per tile (x 3 gates = 48 W_iou rows)
constexpr int NT = 256;         // 4 K slices (alternating 4-column steps) x 64 threads
constexpr int NTC = 128;        // + 4 warps that only clear (warp-specialised: the GEMM never waits for them)
constexpr int KMAX = 256;       // E == KMAX
constexpr int KST = 64;         // K columns per cp.async group
constexpr int NSTG = KMAX / KST;
static_assert(NSTG == 4, "the wait_group sequence below assumes 4 K groups");
constexpr int KS = KMAX + 4;    // row stride in floats (= 4 mod 32: conflict-free 16-byte column reads)
constexpr size_t SMEM = (size_t)(LM + 3 * LU) * KS * sizeof(float);

// Per-pass clearing folded into the leaf kernel (it runs first in the pass): up to 4 float ranges
// (multiples of 4 floats) are zeroed by a grid-stride loop, and the device pass counter is advanced.
__device__ uint64_t g_leaf_prof[1024 * 8];   // measurement only (VPPS_LEAF_PROF): per-CTA phase stamps
__device__ int g_leaf_prof_on;

// barrier of the NT GEMM threads only (the clearing warps never join it)
__device__ __forceinline__ void gemm_sync() { asm volatile("bar.sync 1, %0;" ::"n"(NT) : "memory"); }

struct PassClear {
    float* ptr[4];
    int64_t n[4];
    uint32_t* epoch;     // dataflow pass counter (tags of this pass), or nullptr
};

template <int E>
__global__ void __launch_bounds__(NT + NTC, 1) vpps_leaf_fwd(const float* __restrict__ W, const float* __restrict__ b,
                                                       const float* __restrict__ inputs, float* pool,
                                                       const uint32_t* __restrict__ leaves, int n_leaf, int H,
                                                       const PassClear pc) {
    static_assert(E == KMAX, "leaf GEMM: E == 256");
    extern __shared__ __align__(16) float lsm[];
    __shared__ uint32_t lrec[LM];
    float* As = lsm;                 // [64 leaves][KS]: x rows
    float* Bs = lsm + LM * KS;       // [48 rows][KS]: W_iou rows g*H + j0 + uu, row index g*16 + uu
    const int tid = threadIdx.x;
    // the dataflow kernel may be scheduled as SMs free up (it waits for this grid with griddepcontrol.wait
    // before reading anything written here)
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    const bool pf = g_leaf_prof_on && tid == 0 && blockIdx.x < 1024;
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
        if (g_leaf_prof_on && tid == NT && blockIdx.x < 1024) g_leaf_prof[blockIdx.x * 8 + 6] = gtimer();
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
    asm volatile("cp.async.wait_group 3;" ::: "memory");
    gemm_sync();
    if (pf) pst[2] = gtimer();
    stage(0);
    asm volatile("cp.async.wait_group 2;" ::: "memory");
    gemm_sync();
    stage(1);
    asm volatile("cp.async.wait_group 1;" ::: "memory");
    gemm_sync();
    stage(2);
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    gemm_sync();
    if (pf) pst[3] = gtimer();
    stage(3);
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

}  // namespace leaf
}  // namespace dev

extern "C" int vpps_leaf_prof(int on, uint64_t* out) {   // measurement tool hook (not in vpps.h)
    if (out) return (int)cudaMemcpyFromSymbol(out, dev::leaf::g_leaf_prof, sizeof(uint64_t) * 1024 * 8);
    return (int)cudaMemcpyToSymbol(dev::leaf::g_leaf_prof_on, &on, sizeof(int));
}

void launch_leaf_fwd(const float* W, const float* b, const float* inputs, float* pool, const uint32_t* leaves,
                     int32_t n_leaf, int32_t H, int32_t E, float* const* zero_ptr, const int64_t* zero_n,
                     uint32_t* epoch, cudaStream_t s) {
    using namespace dev::leaf;
    if (E != KMAX || H % LU) return;   // the cluster / dataflow variants are H = E = 256 (api.cu checks)
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(vpps_leaf_fwd<256>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM);
        attr = true;
    }
    PassClear pc{};
    static const int exp_ = getenv("VPPS_LEAF_EXP") ? atoi(getenv("VPPS_LEAF_EXP")) : 0;   // measurement only
    for (int r = 0; r < 4; ++r) { pc.ptr[r] = zero_ptr ? zero_ptr[r] : nullptr; pc.n[r] = zero_ptr ? zero_n[r] : 0; }
    if (exp_ & 1) for (int r = 0; r < 4; ++r) if (r != 2) pc.n[r] = 0;     // no clearing (but the counters)
    if (exp_ & 2) n_leaf = 0;                                                // clearing only
    pc.epoch = epoch;
    const int tiles = std::max(((n_leaf + LM - 1) / LM) * (H / LU), 148);
    vpps_leaf_fwd<256><<<tiles, NT + NTC, SMEM, s>>>(W, b, inputs, pool, leaves, n_leaf, H, pc);
}

}  // namespace vpps
