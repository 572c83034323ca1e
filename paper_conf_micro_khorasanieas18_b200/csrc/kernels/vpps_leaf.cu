// The leaf level of the binary Tree-LSTM as dense GEMMs (cluster path).
//
// Every leaf of a batch uses the same matrix W_iou on its word vector (words enter the
// Tree-LSTM at the leaves), so level 0 is one real dense GEMM — the case where north_star allows a
// GEMM instead of per-node matrix-vector products.  The recurrent matrices (U_iou, U_fl, U_fr) stay
// register-resident in vpps_cl.  Three kernels:
//   vpps_leaf_gemm<FWD>  pre-activations  A[l][r] = W_iou[r] · x_l        -> leaf record gate slots
//   vpps_leaf_cell       leaf cell        i,o = σ, u = tanh, c = i u, h = o tanh c  (in place)
//   vpps_leaf_gemm<DX>   input gradient   dX[tok_l] += W_iouᵀ g_l          (split-K, L2 reductions)
// FP32 SIMT: 64 x 64 output tiles, 16-deep K stages in shared memory (cp.async), 4 x 4 per thread.
#include "vpps_kernel.cuh"
#include "dev_common.cuh"

namespace vpps {
namespace dev {
namespace leaf {

struct Params {
    const float* W;           // W_iou [3H x E] row-major
    const float* b;           // b_iou [3H]
    const float* inputs;      // [rows x E]
    float* pool;
    float* d_inputs;          // DX only
    const uint32_t* leaves;   // n_leaf x (rec, token)
    int32_t n_leaf, H, E, kchunk;
};

constexpr int BM = 64, BN = 64, BK = 16;

// FWD: C[l][n] = Σ_k x_l[k] W[n][k], K = E, N = 3H, written to pool[rec_l + 2H + n] (i, o, u slots)
// DX : C[l][n] = Σ_k g_l[k] W[k][n], K = 3H (this CTA's k chunk), N = E, added to d_inputs[tok_l][n]
template <bool FWD>
__global__ void __launch_bounds__(256) vpps_leaf_gemm(const Params P) {
    __shared__ __align__(16) float As[2][BM][BK];          // [m][k]
    __shared__ __align__(16) float Bs[2][BK][BN + 4];      // [k][n]
    const int tid = threadIdx.x, H = P.H, E = P.E;
    const int N = FWD ? 3 * H : E;
    const int tiles_n = N / BN, tiles_m = (P.n_leaf + BM - 1) / BM;
    int b = blockIdx.x;
    const int kc = b / (tiles_m * tiles_n);
    b -= kc * tiles_m * tiles_n;
    const int m0 = (b / tiles_n) * BM, n0 = (b % tiles_n) * BN;
    const int K = FWD ? E : 3 * H;
    const int k0 = FWD ? 0 : kc * P.kchunk, k1 = FWD ? K : min(K, k0 + P.kchunk);
    const int ty = tid / 16, tx = tid % 16;
    float acc[4][4];
#pragma unroll
    for (int a = 0; a < 4; ++a)
#pragma unroll
        for (int c = 0; c < 4; ++c) acc[a][c] = 0.f;
    auto stage = [&](int kk, int buf) {
        {   // A: 64 rows x 16 k, one 16-byte piece per thread
            const int m = tid / 4, piece = (tid % 4) * 4, row = m0 + m;
            const float* src = nullptr;
            if (row < P.n_leaf) {
                const uint32_t rec = P.leaves[2 * row], tok = P.leaves[2 * row + 1];
                src = FWD ? P.inputs + (int64_t)tok * E + kk + piece : P.pool + rec + 5 * H + kk + piece;
            }
            cp_async16(&As[buf][m][piece], src ? src : P.pool, src ? 16u : 0u);
        }
        if (FWD) {   // B[k][n] = W[n0 + n][kk + k]: 64 rows of W x 16 k, stored transposed (scalar STS)
            const int n = tid / 4, piece = (tid % 4) * 4;
            const float4 w = __ldg(reinterpret_cast<const float4*>(P.W + (int64_t)(n0 + n) * E + kk + piece));
            Bs[buf][piece + 0][n] = w.x; Bs[buf][piece + 1][n] = w.y;
            Bs[buf][piece + 2][n] = w.z; Bs[buf][piece + 3][n] = w.w;
        } else {     // B[k][n] = W[kk + k][n0 + n]: 16 rows x 64 cols
            const int k = tid / 16, piece = (tid % 16) * 4;
            cp_async16(&Bs[buf][k][piece], P.W + (int64_t)(kk + k) * E + n0 + piece, 16u);
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
    };
    const int steps = (k1 - k0) / BK;
    if (steps > 0) stage(k0, 0);
    for (int s = 0; s < steps; ++s) {
        if (s + 1 < steps) {
            stage(k0 + (s + 1) * BK, (s + 1) & 1);
            asm volatile("cp.async.wait_group 1;" ::: "memory");
        } else {
            asm volatile("cp.async.wait_group 0;" ::: "memory");
        }
        __syncthreads();
        const int buf = s & 1;
#pragma unroll
        for (int k = 0; k < BK; ++k) {
            float av[4];
#pragma unroll
            for (int a = 0; a < 4; ++a) av[a] = As[buf][ty * 4 + a][k];
            const float4 bv = *reinterpret_cast<const float4*>(&Bs[buf][k][tx * 4]);
            const float bb[4] = {bv.x, bv.y, bv.z, bv.w};
#pragma unroll
            for (int a = 0; a < 4; ++a)
#pragma unroll
                for (int c = 0; c < 4; ++c) acc[a][c] = fmaf(av[a], bb[c], acc[a][c]);
        }
        __syncthreads();
    }
#pragma unroll
    for (int a = 0; a < 4; ++a) {
        const int row = m0 + ty * 4 + a;
        if (row >= P.n_leaf) continue;
        const uint32_t rec = P.leaves[2 * row], tok = P.leaves[2 * row + 1];
        const int n = n0 + tx * 4;
        if (FWD) {
            *reinterpret_cast<float4*>(P.pool + rec + 2 * H + n) = make_float4(acc[a][0], acc[a][1], acc[a][2], acc[a][3]);
        } else if (P.d_inputs) {
            red_add<4>(P.d_inputs + (int64_t)tok * E + n, acc[a]);
        }
    }
}

// leaf cell (Tai et al. [5] N-ary leaf): a = pre-activation + b_iou; c = σ(a_i) tanh(a_u); h = σ(a_o) tanh(c)
__global__ void vpps_leaf_cell(const Params P) {
    const int H = P.H;
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (int64_t)P.n_leaf * H;
         i += (int64_t)gridDim.x * blockDim.x) {
        const int l = (int)(i / H), j = (int)(i - (int64_t)l * H);
        float* r = P.pool + P.leaves[2 * l];
        const float ig = sigm(r[2 * H + j] + __ldg(P.b + j));
        const float og = sigm(r[3 * H + j] + __ldg(P.b + H + j));
        const float ug = tanhf(r[4 * H + j] + __ldg(P.b + 2 * H + j));
        const float c = ig * ug;
        r[j] = og * tanhf(c);
        r[H + j] = c;
        r[2 * H + j] = ig;
        r[3 * H + j] = og;
        r[4 * H + j] = ug;
    }
}

}  // namespace leaf
}  // namespace dev

void launch_leaf_fwd(const float* W, const float* b, const float* inputs, float* pool, const uint32_t* leaves,
                     int32_t n_leaf, int32_t H, int32_t E, cudaStream_t s) {
    using namespace dev::leaf;
    if (n_leaf <= 0) return;
    Params p{W, b, inputs, pool, nullptr, leaves, n_leaf, H, E, 0};
    const int tiles = ((n_leaf + BM - 1) / BM) * (3 * H / BN);
    vpps_leaf_gemm<true><<<tiles, 256, 0, s>>>(p);
    vpps_leaf_cell<<<(int)std::min<int64_t>(1184, ((int64_t)n_leaf * H + 255) / 256), 256, 0, s>>>(p);
}

void launch_leaf_dx(const float* W, const float* pool, float* d_inputs, const uint32_t* leaves, int32_t n_leaf,
                    int32_t H, int32_t E, cudaStream_t s) {
    using namespace dev::leaf;
    if (n_leaf <= 0 || !d_inputs) return;
    const int kchunk = 128;
    Params p{W, nullptr, nullptr, const_cast<float*>(pool), d_inputs, leaves, n_leaf, H, E, kchunk};
    const int tiles = ((n_leaf + BM - 1) / BM) * (E / BN) * ((3 * H + kchunk - 1) / kchunk);
    vpps_leaf_gemm<false><<<tiles, 256, 0, s>>>(p);
}

}  // namespace vpps
