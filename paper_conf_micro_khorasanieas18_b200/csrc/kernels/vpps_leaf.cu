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
// Tile: 32 leaves x 32 hidden units x 3 gates (i, o, u of the same units, so the cell runs in the
// epilogue).  The whole K range of the tile's 128 rows is staged with one batch of cp.async (the GEMM is
// small and DRAM-latency bound after the L2 flush, so one round trip beats a K pipeline); 512 threads =
// four K quarters of 128; each thread owns 4 leaves x 2 units x 3 gates and reads 16-byte K slices.
// The input-table gradient dX = W_iouᵀ g_leaf is a job of the gradient GEMM (vpps_dw_gemm, vpps_cluster.cu).
// Requires E <= KMAX and H % 32 == 0 (the cluster variants are H = E = 256).
#include "vpps_kernel.cuh"
#include "dev_common.cuh"

namespace vpps {
namespace dev {
namespace leaf {

constexpr int LM = 32;          // leaves per tile
constexpr int LU = 32;          // hidden units per tile (x 3 gates)
constexpr int NT = 512;
constexpr int KMAX = 256;       // E <= KMAX: the whole K range is staged at once (one DRAM round trip)
constexpr int KS = KMAX + 4;    // row stride in floats (≡ 4 mod 32: conflict-free 16-byte column reads)
constexpr size_t SMEM = (size_t)(LM + 3 * LU) * KS * sizeof(float);

__global__ void __launch_bounds__(NT, 1) vpps_leaf_fwd(const float* __restrict__ W, const float* __restrict__ b,
                                                    const float* __restrict__ inputs, float* pool,
                                                    const uint32_t* __restrict__ leaves, int n_leaf, int H, int E) {
    extern __shared__ __align__(16) float lsm[];
    float* As = lsm;                 // [32 leaves][KS]: x rows
    float* Bs = lsm + LM * KS;       // [96 rows][KS]: W_iou rows g*H + j0 + uu, row index g*32 + uu
    const int tid = threadIdx.x;
    const int tiles_u = H / LU;
    const int l0 = (blockIdx.x / tiles_u) * LM, j0 = (blockIdx.x % tiles_u) * LU;
    // stage everything: 128 rows x E floats, 16-byte cp.async pieces, zero-filled past the last leaf
    const int q = E / 4;
    for (int i = tid; i < (LM + 3 * LU) * q; i += NT) {
        const int row = i / q, c = (i - row * q) * 4;
        const float* src = nullptr;
        if (row < LM) {
            const int l = l0 + row;
            if (l < n_leaf) src = inputs + (int64_t)leaves[2 * l + 1] * E + c;
        } else {
            const int r = row - LM, g = r / LU, uu = r % LU;
            src = W + (int64_t)(g * H + j0 + uu) * E + c;
        }
        cp_async16(lsm + row * KS + c, src ? src : W, src ? 16u : 0u);
    }
    cp_async_wait_all();
    __syncthreads();
    // 4 K quarters x 128 threads; a thread owns 4 leaves x 2 units x 3 gates (24 accumulators): per 4-wide K
    // step 4 + 6 LDS.128 feed 96 FMA, so the FMA pipe, not shared memory, is the limit
    const int part = tid >> 7, tt = tid & 127, lq = tt >> 4, up = tt & 15;
    float acc[4][3][2];
#pragma unroll
    for (int a = 0; a < 4; ++a)
#pragma unroll
        for (int g = 0; g < 3; ++g) acc[a][g][0] = acc[a][g][1] = 0.f;
    const int kq = E / 4, kb = part * kq;
    const float* ap = As + (4 * lq) * KS + kb;
    const float* bw = Bs + up * KS + kb;
#pragma unroll 2
    for (int k = 0; k < kq; k += 4) {
        float4 x[4];
#pragma unroll
        for (int a = 0; a < 4; ++a) x[a] = *reinterpret_cast<const float4*>(ap + a * KS + k);
#pragma unroll
        for (int g = 0; g < 3; ++g)
#pragma unroll
            for (int c = 0; c < 2; ++c) {
                const float4 w = *reinterpret_cast<const float4*>(bw + (g * LU + 16 * c) * KS + k);
#pragma unroll
                for (int a = 0; a < 4; ++a)
                    acc[a][g][c] = fmaf(x[a].x, w.x, fmaf(x[a].y, w.y, fmaf(x[a].z, w.z, fmaf(x[a].w, w.w, acc[a][g][c]))));
            }
    }
    __syncthreads();
    float* red = lsm;                // [3 parts][128][25]: partial sums of K quarters 1..3 (aliases the staging)
    if (part > 0) {
        float* o = red + ((part - 1) * 128 + tt) * 25;
#pragma unroll
        for (int a = 0; a < 4; ++a)
#pragma unroll
            for (int g = 0; g < 3; ++g) { o[a * 6 + g * 2] = acc[a][g][0]; o[a * 6 + g * 2 + 1] = acc[a][g][1]; }
    }
    __syncthreads();
    if (part > 0) return;
#pragma unroll
    for (int p = 0; p < 3; ++p) {
        const float* o = red + (p * 128 + tt) * 25;
#pragma unroll
        for (int a = 0; a < 4; ++a)
#pragma unroll
            for (int g = 0; g < 3; ++g) { acc[a][g][0] += o[a * 6 + g * 2]; acc[a][g][1] += o[a * 6 + g * 2 + 1]; }
    }
    float bb[3][2];
#pragma unroll
    for (int g = 0; g < 3; ++g)
#pragma unroll
        for (int c = 0; c < 2; ++c) bb[g][c] = __ldg(b + g * H + j0 + up + 16 * c);
#pragma unroll
    for (int a = 0; a < 4; ++a) {
        const int l = l0 + 4 * lq + a;
        if (l >= n_leaf) continue;
        float* r = pool + leaves[2 * l];
#pragma unroll
        for (int c = 0; c < 2; ++c) {
            const int j = j0 + up + 16 * c;
            const float ig = sigm(acc[a][0][c] + bb[0][c]), og = sigm(acc[a][1][c] + bb[1][c]);
            const float ug = tanhf(acc[a][2][c] + bb[2][c]);
            const float cc = ig * ug;
            r[j] = og * tanhf(cc);
            r[H + j] = cc;
            r[2 * H + j] = ig;
            r[3 * H + j] = og;
            r[4 * H + j] = ug;
        }
    }
}

}  // namespace leaf
}  // namespace dev

void launch_leaf_fwd(const float* W, const float* b, const float* inputs, float* pool, const uint32_t* leaves,
                     int32_t n_leaf, int32_t H, int32_t E, cudaStream_t s) {
    using namespace dev::leaf;
    if (n_leaf <= 0) return;
    static bool attr = false;
    if (!attr) {
        cudaFuncSetAttribute(vpps_leaf_fwd, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM);
        attr = true;
    }
    const int tiles = ((n_leaf + LM - 1) / LM) * (H / LU);
    vpps_leaf_fwd<<<tiles, NT, SMEM, s>>>(W, b, inputs, pool, leaves, n_leaf, H, E);
}

}  // namespace vpps
