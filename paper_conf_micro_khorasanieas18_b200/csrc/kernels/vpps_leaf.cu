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
// Tile: 16 leaves x 16 hidden units x 3 gates (i, o, u of the same units, so the cell runs in the
// epilogue); ~370 CTAs, 3 per SM.  The whole K range of the tile's 64 rows is staged with one batch of
// cp.async (small GEMM, latency bound: one round trip beats a K pipeline); 128 threads = four K quarters
// of 32; each thread owns 4 leaves x 2 units x 3 gates and reads 16-byte K slices.
// The input-table gradient dX = W_iouᵀ g_leaf is a job of the gradient GEMM (vpps_dw_gemm, vpps_cluster.cu).
// Requires E <= KMAX and H % 32 == 0 (the cluster variants are H = E = 256).
#include <algorithm>
#include "vpps_kernel.cuh"
#include "dev_common.cuh"

namespace vpps {
namespace dev {
namespace leaf {

constexpr int LM = 16;          // leaves per tile
constexpr int LU = 16;          // hidden units per tile (x 3 gates = 48 W_iou rows)
constexpr int NT = 128;         // 4 K quarters x 32 threads
constexpr int KMAX = 256;       // E <= KMAX: the whole K range is staged at once (one round trip)
constexpr int KS = KMAX + 4;    // row stride in floats (≡ 4 mod 32: conflict-free 16-byte column reads)
constexpr size_t SMEM = (size_t)(LM + 3 * LU) * KS * sizeof(float);

// Per-pass clearing folded into the leaf kernel (it runs first in the pass): up to 4 float ranges
// (multiples of 4 floats) are zeroed by a grid-stride loop, and the device pass counter is advanced.
struct PassClear {
    float* ptr[4];
    int64_t n[4];
    uint32_t* epoch;     // dataflow pass counter (tags of this pass), or nullptr
};

template <int E>
__global__ void __launch_bounds__(NT, 3) vpps_leaf_fwd(const float* __restrict__ W, const float* __restrict__ b,
                                                       const float* __restrict__ inputs, float* pool,
                                                       const uint32_t* __restrict__ leaves, int n_leaf, int H,
                                                       const PassClear pc) {
    static_assert(E <= KMAX && E % 16 == 0, "leaf GEMM: E <= 256");
    extern __shared__ __align__(16) float lsm[];
    __shared__ uint32_t lrec[LM], ltok[LM];
    float* As = lsm;                 // [16 leaves][KS]: x rows
    float* Bs = lsm + LM * KS;       // [48 rows][KS]: W_iou rows g*H + j0 + uu, row index g*16 + uu
    const int tid = threadIdx.x;
    if (pc.epoch && blockIdx.x == 0 && tid == 0) {
        uint32_t e = *pc.epoch + 1;
        *pc.epoch = e ? e : 1u;                                   // 0 marks never-written slots
    }
    {
        const int64_t stride = (int64_t)gridDim.x * NT;
        for (int r = 0; r < 4; ++r) {
            float4* p = reinterpret_cast<float4*>(pc.ptr[r]);
            const int64_t n4 = pc.ptr[r] ? pc.n[r] / 4 : 0;
            for (int64_t i = (int64_t)blockIdx.x * NT + tid; i < n4; i += stride) p[i] = make_float4(0.f, 0.f, 0.f, 0.f);
        }
    }
    const int tiles_u = H / LU;
    const int l0 = (blockIdx.x / tiles_u) * LM, j0 = (blockIdx.x % tiles_u) * LU;
    if (l0 >= n_leaf) return;                                      // clearing-only CTA
    if (tid < LM) {
        const int l = l0 + tid;
        lrec[tid] = l < n_leaf ? leaves[2 * l] : 0u;
        ltok[tid] = l < n_leaf ? leaves[2 * l + 1] : 0xFFFFFFFFu;
    }
    // W rows first (independent of the leaf list), then the x rows
    constexpr int Q = E / 4;                       // 16-byte pieces per row
    for (int i = tid; i < 3 * LU * Q; i += NT) {
        const int r = i / Q, c = (i % Q) * 4, g = r / LU, uu = r % LU;
        cp_async16(Bs + r * KS + c, W + (int64_t)(g * H + j0 + uu) * E + c, 16u);
    }
    __syncthreads();
    for (int i = tid; i < LM * Q; i += NT) {
        const int r = i / Q, c = (i % Q) * 4;
        const uint32_t tok = ltok[r];
        const bool ok = tok != 0xFFFFFFFFu;
        cp_async16(As + r * KS + c, ok ? inputs + (int64_t)tok * E + c : W, ok ? 16u : 0u);
    }
    cp_async_wait_all();
    __syncthreads();
    // a thread owns 4 leaves x 2 units x 3 gates (24 accumulators) over one K quarter: per 4-wide K step
    // 4 + 6 LDS.128 feed 96 FMA
    const int part = tid >> 5, tt = tid & 31, lq = tt >> 3, up = tt & 7;   // leaves 4lq..+3, units up, up+8
    float acc[4][3][2];
#pragma unroll
    for (int a = 0; a < 4; ++a)
#pragma unroll
        for (int g = 0; g < 3; ++g) acc[a][g][0] = acc[a][g][1] = 0.f;
    constexpr int KQ = E / 4;
    const float* ap = As + (4 * lq) * KS + part * KQ;
    const float* bw = Bs + up * KS + part * KQ;
#pragma unroll 2
    for (int k = 0; k < KQ; k += 4) {
        float4 x[4];
#pragma unroll
        for (int a = 0; a < 4; ++a) x[a] = *reinterpret_cast<const float4*>(ap + a * KS + k);
#pragma unroll
        for (int g = 0; g < 3; ++g)
#pragma unroll
            for (int c = 0; c < 2; ++c) {
                const float4 w = *reinterpret_cast<const float4*>(bw + (g * LU + 8 * c) * KS + k);
#pragma unroll
                for (int a = 0; a < 4; ++a)
                    acc[a][g][c] = fmaf(x[a].x, w.x, fmaf(x[a].y, w.y, fmaf(x[a].z, w.z, fmaf(x[a].w, w.w, acc[a][g][c]))));
            }
    }
    __syncthreads();
    // reduce the 4 K quarters through shared memory; warp `part` then finishes leaf 4lq + part
    float* red = lsm;                // [4 parts][32][25] (aliases the staging)
    {
        float* o = red + (part * 32 + tt) * 25;
#pragma unroll
        for (int a = 0; a < 4; ++a)
#pragma unroll
            for (int g = 0; g < 3; ++g) { o[a * 6 + g * 2] = acc[a][g][0]; o[a * 6 + g * 2 + 1] = acc[a][g][1]; }
    }
    __syncthreads();
    const int a = part, li = 4 * lq + a;
    if (l0 + li >= n_leaf) return;
    float pre[3][2] = {{0.f, 0.f}, {0.f, 0.f}, {0.f, 0.f}};
#pragma unroll
    for (int p = 0; p < 4; ++p) {
        const float* o = red + (p * 32 + tt) * 25 + a * 6;
#pragma unroll
        for (int g = 0; g < 3; ++g) { pre[g][0] += o[g * 2]; pre[g][1] += o[g * 2 + 1]; }
    }
    float* r = pool + lrec[li];
#pragma unroll
    for (int c = 0; c < 2; ++c) {
        const int j = j0 + up + 8 * c;
        const float ig = fsigm(pre[0][c] + __ldg(b + j)), og = fsigm(pre[1][c] + __ldg(b + H + j));
        const float ug = ftanh(pre[2][c] + __ldg(b + 2 * H + j));
        const float cc = ig * ug;
        r[j] = og * ftanh(cc);
        r[H + j] = cc;
        r[2 * H + j] = ig;
        r[3 * H + j] = og;
        r[4 * H + j] = ug;
    }
}

}  // namespace leaf
}  // namespace dev

void launch_leaf_fwd(const float* W, const float* b, const float* inputs, float* pool, const uint32_t* leaves,
                     int32_t n_leaf, int32_t H, int32_t E, float* const* zero_ptr, const int64_t* zero_n,
                     uint32_t* epoch, cudaStream_t s) {
    using namespace dev::leaf;
    if (E != 256 || H % LU) return;   // the cluster / dataflow variants are H = E = 256 (api.cu checks)
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(vpps_leaf_fwd<256>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM);
        attr = true;
    }
    PassClear pc{};
    for (int r = 0; r < 4; ++r) { pc.ptr[r] = zero_ptr ? zero_ptr[r] : nullptr; pc.n[r] = zero_ptr ? zero_n[r] : 0; }
    pc.epoch = epoch;
    const int tiles = std::max(((n_leaf + LM - 1) / LM) * (H / LU), 148);
    vpps_leaf_fwd<256><<<tiles, NT, SMEM, s>>>(W, b, inputs, pool, leaves, n_leaf, H, pc);
}

}  // namespace vpps
