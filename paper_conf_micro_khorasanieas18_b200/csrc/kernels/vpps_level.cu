// Level-synchronous path of the binary Tree-LSTM for hidden sizes whose recurrent weights do not fit a
// 16-CTA replica group's registers (config 5: H = E = 1024, 33.5 MB of U_iou, U_fl, U_fr).
//
// The paper's fallback for weight gradients that do not fit on chip ("concatenate all the left
// hand side and all the right hand side tensors that participate in the outer-product for each weight
// matrix, and use dense matrix-matrix multiplication") is applied to every matrix use: per level, the
// children's [h_l; h_r] rows are gathered and multiplied by the weights as one dense GEMM (the level
// batches "enough same-parameter nodes to form a real dense GEMM", north_star), the cell runs as a fused
// elementwise pass, and the backward level multiplies the gate gradients by the same weights.  The weights
// (33.5 MB) stay resident in the 126 MB L2 across the levels of a pass, so DRAM still reads them about once
// per pass; this is a deliberate deviation from register residency.  The dense products are
// plain FP32 GEMMs (cuBLAS SGEMM, no TF32); gathers, cells, heads, scatters and bias gradients are the
// kernels below.  Pool records and adjoint blocks follow SPEC_SCRIPT §S7 (binary leaf [h c i o u | g_i g_o
// g_u], internal [h c i o u f_l f_r | g_i g_o g_u g_fl g_fr], head [p(C) loss], adj [dh | dc]).
#include <cublas_v2.h>
#include <algorithm>
#include <cstdio>
#include "vpps_kernel.cuh"
#include "dev_common.cuh"

namespace vpps {
namespace dev {
namespace lv {

constexpr uint32_t NONE = 0xFFFFFFFFu;

// X[r][0:E] = inputs[token(r)] (zeros for a leaf without a token)
__global__ void gather_leaf(const float* __restrict__ inputs, const uint32_t* __restrict__ leaf, int n, int E,
                            float* __restrict__ X) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, total = (int64_t)n * (E / 4);
    if (i >= total) return;
    const int r = (int)(i / (E / 4)), c = (int)(i % (E / 4)) * 4;
    const uint32_t tok = leaf[3 * r + 2];
    const float4 v = tok == NONE ? make_float4(0.f, 0.f, 0.f, 0.f)
                                 : __ldg(reinterpret_cast<const float4*>(inputs + (int64_t)tok * E + c));
    *reinterpret_cast<float4*>(X + (int64_t)r * E + c) = v;
}

// leaf cell: a = Z + b_iou; i, o = σ, u = tanh; c = i u; h = o tanh c -> record [h c i o u]
__global__ void leaf_cell(const float* __restrict__ Z, const float* __restrict__ b_iou,
                          const uint32_t* __restrict__ leaf, int n, int H, float* pool) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    const float* z = Z + (int64_t)r * 3 * H;
    const float i = sigm(z[j] + b_iou[j]), o = sigm(z[H + j] + b_iou[H + j]), u = tanhf(z[2 * H + j] + b_iou[2 * H + j]);
    const float c = i * u;
    float* rec = pool + leaf[3 * r];
    rec[j] = o * tanhf(c);
    rec[H + j] = c;
    rec[2 * H + j] = i;
    rec[3 * H + j] = o;
    rec[4 * H + j] = u;
}

// X[r] = [h(rec_l); h(rec_r)] for the internal nodes of one level
__global__ void gather_int(const float* __restrict__ pool, const uint32_t* __restrict__ nodes, int n, int H,
                           float* __restrict__ X) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, q = 2 * H / 4, total = (int64_t)n * q;
    if (i >= total) return;
    const int r = (int)(i / q), c = (int)(i % q) * 4;
    const uint32_t* e = nodes + 6 * r;
    const float* src = c < H ? pool + e[1] + c : pool + e[2] + (c - H);
    *reinterpret_cast<float4*>(X + (int64_t)r * 2 * H + c) = __ldcg(reinterpret_cast<const float4*>(src));
}

// internal cell (PAPER's Tree-LSTM workload, [5] eqs. 9-14 with N = 2, diagonal forget couplings):
// a_iou = Z[:, 0:3H] + b_iou, f_l = σ(Z[:, 3H:4H] + b_f), f_r = σ(Z[:, 4H:5H] + b_f),
// c = i u + f_l c_l + f_r c_r, h = o tanh c -> record [h c i o u f_l f_r]
__global__ void int_cell(const float* __restrict__ Z, const float* __restrict__ b_iou, const float* __restrict__ b_f,
                         const uint32_t* __restrict__ nodes, int n, int H, float* pool) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    const uint32_t* e = nodes + 6 * r;
    const float* z = Z + (int64_t)r * 5 * H;
    const float i = sigm(z[j] + b_iou[j]), o = sigm(z[H + j] + b_iou[H + j]), u = tanhf(z[2 * H + j] + b_iou[2 * H + j]);
    const float fl = sigm(z[3 * H + j] + b_f[j]), fr = sigm(z[4 * H + j] + b_f[j]);
    const float c = i * u + fl * __ldcg(pool + e[1] + H + j) + fr * __ldcg(pool + e[2] + H + j);
    float* rec = pool + e[0];
    rec[j] = o * tanhf(c);
    rec[H + j] = c;
    rec[2 * H + j] = i;
    rec[3 * H + j] = o;
    rec[4 * H + j] = u;
    rec[5 * H + j] = fl;
    rec[6 * H + j] = fr;
}

// loss heads (L42), one CTA per head: z = W_out h + b_out, softmax-NLL into the record and the summed loss
// (L205); dz = p - onehot(y): dW_out += dz hᵀ, db_out += dz (atomics), the cell's dh += W_outᵀ dz
__global__ void heads(const float* __restrict__ Wo, const float* __restrict__ bo, const uint32_t* __restrict__ hl,
                      int H, int C, float* pool, int64_t loss_word, float* dWo, float* dbo) {
    extern __shared__ float zsh[];      // [C]
    const uint32_t* e = hl + 4 * blockIdx.x;
    const float* h = pool + e[1];
    const int y = (int)e[3];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nw = blockDim.x >> 5;
    for (int c = warp; c < C; c += nw) {
        float s = 0.f;
        for (int k = lane; k < H; k += 32) s = fmaf(Wo[(int64_t)c * H + k], __ldcg(h + k), s);
        s = warp_sum(s);
        if (lane == 0) zsh[c] = s + bo[c];
    }
    __syncthreads();
    if (warp == 0) {
        float m = -INFINITY;
        for (int c = lane; c < C; c += 32) m = fmaxf(m, zsh[c]);
        m = warp_max(m);
        float se = 0.f;
        for (int c = lane; c < C; c += 32) se += expf(zsh[c] - m);
        const float lse = m + logf(warp_sum(se));
        const float zy = zsh[y];
        __syncwarp();
        for (int c = lane; c < C; c += 32) {
            const float p = expf(zsh[c] - lse);
            pool[e[0] + c] = p;
            zsh[c] = p - (c == y ? 1.f : 0.f);       // dz = softmax - onehot(y)
        }
        if (lane == 0) {
            pool[e[0] + C] = lse - zy;
            atomicAdd(pool + loss_word, lse - zy);
        }
    }
    __syncthreads();
    for (int c = threadIdx.x; c < C; c += blockDim.x) atomicAdd(dbo + c, zsh[c]);
    for (int64_t i = threadIdx.x; i < (int64_t)C * H; i += blockDim.x) {
        const int c = (int)(i / H), k = (int)(i % H);
        atomicAdd(dWo + i, zsh[c] * __ldcg(h + k));
    }
    for (int k = threadIdx.x; k < H; k += blockDim.x) {
        float s = 0.f;
        for (int c = 0; c < C; ++c) s = fmaf(Wo[(int64_t)c * H + k], zsh[c], s);
        atomicAdd(pool + e[2] + k, s);     // dh of the labelled cell (adj block)
    }
}

// internal cell backward (c.2b): given dh, dc (adj) -> gate gradients g = [g_i g_o g_u g_fl g_fr] into the
// record and the level's G rows; the children's dc (each child has this node as its only parent)
__global__ void int_bwd(const uint32_t* __restrict__ nodes, int n, int H, float* pool, float* __restrict__ G) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    const uint32_t* e = nodes + 6 * r;
    const float* rec = pool + e[0];
    const float dh = __ldcg(pool + e[3] + j), dc = __ldcg(pool + e[3] + H + j);
    const float c = rec[H + j], i = rec[2 * H + j], o = rec[3 * H + j], u = rec[4 * H + j];
    const float fl = rec[5 * H + j], fr = rec[6 * H + j];
    const float cl = __ldcg(pool + e[1] + H + j), cr = __ldcg(pool + e[2] + H + j);
    const float th = tanhf(c);
    const float chat = dc + dh * o * (1.f - th * th);
    const float g[5] = {chat * u * i * (1.f - i), dh * th * o * (1.f - o), chat * i * (1.f - u * u),
                        chat * cl * fl * (1.f - fl), chat * cr * fr * (1.f - fr)};
    float* gr = pool + e[0] + 7 * H;
    float* Gr = G + (int64_t)r * 5 * H;
#pragma unroll
    for (int k = 0; k < 5; ++k) { gr[k * H + j] = g[k]; Gr[k * H + j] = g[k]; }
    pool[e[4] + H + j] = chat * fl;
    pool[e[5] + H + j] = chat * fr;
}

// children's dh += DX rows (left half -> child l, right half -> child r); unique parent: plain adds
__global__ void scatter_dh(const float* __restrict__ DX, const uint32_t* __restrict__ nodes, int n, int H, float* pool) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * 2 * H) return;
    const int r = (int)(t / (2 * H)), c = (int)(t % (2 * H));
    const uint32_t* e = nodes + 6 * r;
    float* dst = c < H ? pool + e[4] + c : pool + e[5] + (c - H);
    *dst += DX[t];
}

// leaf cell backward -> g = [g_i g_o g_u] into the record and G_leaf
__global__ void leaf_bwd(const uint32_t* __restrict__ leaf, int n, int H, float* pool, float* __restrict__ G) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    const uint32_t* e = leaf + 3 * r;
    const float* rec = pool + e[0];
    const float dh = __ldcg(pool + e[1] + j), dc = __ldcg(pool + e[1] + H + j);
    const float c = rec[H + j], i = rec[2 * H + j], o = rec[3 * H + j], u = rec[4 * H + j];
    const float th = tanhf(c);
    const float chat = dc + dh * o * (1.f - th * th);
    const float g[3] = {chat * u * i * (1.f - i), dh * th * o * (1.f - o), chat * i * (1.f - u * u)};
    float* gr = pool + e[0] + 5 * H;
    float* Gr = G + (int64_t)r * 3 * H;
#pragma unroll
    for (int k = 0; k < 3; ++k) { gr[k * H + j] = g[k]; Gr[k * H + j] = g[k]; }
}

// dX[token] += DXL rows (duplicate tokens: atomics)
__global__ void scatter_dx(const float* __restrict__ DXL, const uint32_t* __restrict__ leaf, int n, int E, float* dX) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * E) return;
    const int r = (int)(t / E), c = (int)(t % E);
    const uint32_t tok = leaf[3 * r + 2];
    if (tok != NONE) atomicAdd(dX + (int64_t)tok * E + c, DXL[t]);
}

// bias gradients: db_iou[k] = Σ_rows G_int[:, k] + Σ_rows G_leaf[:, k] (k < 3H), db_f[j] = Σ G_int[:, 3H+j] + G_int[:, 4H+j]
__global__ void bias_grads(const float* __restrict__ Gi, int ni, const float* __restrict__ Gl, int nl, int H,
                           float* db_iou, float* db_f) {
    const int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= 4 * H) return;
    float s = 0.f;
    if (k < 3 * H) {
        for (int r = 0; r < ni; ++r) s += Gi[(int64_t)r * 5 * H + k];
        for (int r = 0; r < nl; ++r) s += Gl[(int64_t)r * 3 * H + k];
        db_iou[k] = s;
    } else {
        const int j = k - 3 * H;
        for (int r = 0; r < ni; ++r) s += Gi[(int64_t)r * 5 * H + 3 * H + j] + Gi[(int64_t)r * 5 * H + 4 * H + j];
        db_f[j] = s;
    }
}

}  // namespace lv
}  // namespace dev

// ---- host orchestration ------------------------------------------------------------------------

// Row-major C[M x N] = alpha op(A) op(B) + beta C (A: M x K, or K x M when ta; B: K x N, or N x K when tb)
static cublasStatus_t gemm_rm(cublasHandle_t h, bool ta, bool tb, int M, int N, int K, const float* A, int lda,
                              const float* B, int ldb, float* C, int ldc, float beta) {
    const float alpha = 1.f;
    if (M <= 0 || N <= 0) return CUBLAS_STATUS_SUCCESS;
    if (K <= 0) return CUBLAS_STATUS_SUCCESS;      // only dW products with no nodes: grads stay zero
    return cublasSgemm(h, tb ? CUBLAS_OP_T : CUBLAS_OP_N, ta ? CUBLAS_OP_T : CUBLAS_OP_N, N, M, K, &alpha, B, ldb,
                       A, lda, &beta, C, ldc);
}

struct LevelBufs {
    float *X_leaf = nullptr, *X_int = nullptr, *Z = nullptr, *G_int = nullptr, *G_leaf = nullptr, *DX = nullptr;
    int64_t cap_leaf = 0, cap_int = 0;
};

static bool grow(float** p, int64_t* cap, int64_t need) {
    if (need <= *cap) return true;
    if (*p) cudaFree(*p);
    *p = nullptr;
    const int64_t c = need + need / 4 + 1024;
    if (cudaMalloc(p, c * sizeof(float)) != cudaSuccess) return false;
    *cap = c;
    return true;
}

struct LevelCtx {
    cublasHandle_t blas = nullptr;
    LevelBufs b;
    int64_t cap_X_leaf = 0, cap_X_int = 0, cap_Z = 0, cap_G_int = 0, cap_G_leaf = 0, cap_DX = 0;
};

void* level_ctx_create() {
    LevelCtx* c = new LevelCtx;
    if (cublasCreate(&c->blas) != CUBLAS_STATUS_SUCCESS) { delete c; return nullptr; }
    cublasSetMathMode(c->blas, CUBLAS_PEDANTIC_MATH);     // plain FP32 (no TF32, no emulation)
    return c;
}

void level_ctx_destroy(void* p) {
    LevelCtx* c = static_cast<LevelCtx*>(p);
    if (!c) return;
    if (c->blas) cublasDestroy(c->blas);
    float* bufs[] = {c->b.X_leaf, c->b.X_int, c->b.Z, c->b.G_int, c->b.G_leaf, c->b.DX};
    for (float* q : bufs) if (q) cudaFree(q);
    delete c;
}

static inline unsigned nblk(int64_t n, int t = 256) { return (unsigned)((n + t - 1) / t); }

// One forward + backward pass (+ dW, bias and head gradients into grads, which the caller zeroed; dX into
// d_inputs, zeroed by the caller).  Returns a CUDA / cuBLAS error code (0 = ok).
int level_pass(void* ctx_, const float* params, const int64_t* off, float* grads, float* pool, const float* inputs,
               float* d_inputs, const uint32_t* d_blob, int64_t lv_int, int64_t lv_leaf, int64_t lv_head,
               const int32_t* lv_start, int32_t L, int64_t n_int, int64_t n_leaf, int64_t n_head, int32_t H,
               int32_t E, int32_t C, int64_t loss_word, cudaStream_t s) {
    using namespace dev::lv;
    LevelCtx* c = static_cast<LevelCtx*>(ctx_);
    cublasSetStream(c->blas, s);
    const int64_t zrows = std::max<int64_t>(n_leaf * 3 * H, n_int * 5 * H);
    if (!grow(&c->b.X_leaf, &c->cap_X_leaf, std::max<int64_t>(n_leaf * E, 4)) ||
        !grow(&c->b.X_int, &c->cap_X_int, std::max<int64_t>(n_int * 2 * H, 4)) ||
        !grow(&c->b.Z, &c->cap_Z, std::max<int64_t>(zrows, 4)) ||
        !grow(&c->b.G_int, &c->cap_G_int, std::max<int64_t>(n_int * 5 * H, 4)) ||
        !grow(&c->b.G_leaf, &c->cap_G_leaf, std::max<int64_t>(n_leaf * 3 * H, 4)) ||
        !grow(&c->b.DX, &c->cap_DX, std::max<int64_t>(std::max<int64_t>(n_int * 2 * H, n_leaf * E), 4)))
        return (int)cudaErrorMemoryAllocation;
    const float* W_iou = params + off[0];
    const float* U_iou = params + off[1];
    const float* U_fl = params + off[2];
    const float* U_fr = params + off[3];
    const float* W_out = params + off[4];
    const float* b_iou = params + off[5];
    const float* b_f = params + off[6];
    const float* b_out = params + off[7];
    const uint32_t* ints = d_blob + lv_int;
    const uint32_t* leaves = d_blob + lv_leaf;
    const uint32_t* hl = d_blob + lv_head;
    float *Xl = c->b.X_leaf, *Xi = c->b.X_int, *Z = c->b.Z, *Gi = c->b.G_int, *Gl = c->b.G_leaf, *DX = c->b.DX;
    cublasStatus_t st = CUBLAS_STATUS_SUCCESS;
#define BL(call) do { st = (call); if (st != CUBLAS_STATUS_SUCCESS) return 1000 + (int)st; } while (0)
    // ---- forward: leaves (level 0) as one GEMM, then every internal level ----
    if (n_leaf > 0) {
        gather_leaf<<<nblk(n_leaf * (E / 4)), 256, 0, s>>>(inputs, leaves, (int)n_leaf, E, Xl);
        BL(gemm_rm(c->blas, false, true, (int)n_leaf, 3 * H, E, Xl, E, W_iou, E, Z, 3 * H, 0.f));
        leaf_cell<<<nblk(n_leaf * H), 256, 0, s>>>(Z, b_iou, leaves, (int)n_leaf, H, pool);
    }
    for (int32_t l = 1; l <= L; ++l) {
        const int64_t r0 = lv_start[l], n = lv_start[l + 1] - r0;
        if (n <= 0) continue;
        float* X = Xi + r0 * 2 * H;
        gather_int<<<nblk(n * (2 * H / 4)), 256, 0, s>>>(pool, ints + 6 * r0, (int)n, H, X);
        BL(gemm_rm(c->blas, false, true, (int)n, 3 * H, 2 * H, X, 2 * H, U_iou, 2 * H, Z, 5 * H, 0.f));
        BL(gemm_rm(c->blas, false, true, (int)n, H, H, X, 2 * H, U_fl, H, Z + 3 * H, 5 * H, 0.f));
        BL(gemm_rm(c->blas, false, true, (int)n, H, H, X + H, 2 * H, U_fr, H, Z + 4 * H, 5 * H, 0.f));
        int_cell<<<nblk(n * H), 256, 0, s>>>(Z, b_iou, b_f, ints + 6 * r0, (int)n, H, pool);
    }
    // ---- loss heads: forward and backward (they feed nothing forward) ----
    if (n_head > 0)
        heads<<<(unsigned)n_head, 256, C * sizeof(float), s>>>(W_out, b_out, hl, H, C, pool, loss_word, grads + off[4],
                                                             grads + off[7]);
    // ---- backward: internal levels L .. 1, then the leaves ----
    for (int32_t l = L; l >= 1; --l) {
        const int64_t r0 = lv_start[l], n = lv_start[l + 1] - r0;
        if (n <= 0) continue;
        float* G = Gi + r0 * 5 * H;
        int_bwd<<<nblk(n * H), 256, 0, s>>>(ints + 6 * r0, (int)n, H, pool, G);
        // [dh_l; dh_r] = U_iouᵀ g_iou, dh_l += U_flᵀ g_fl, dh_r += U_frᵀ g_fr
        BL(gemm_rm(c->blas, false, false, (int)n, 2 * H, 3 * H, G, 5 * H, U_iou, 2 * H, DX, 2 * H, 0.f));
        BL(gemm_rm(c->blas, false, false, (int)n, H, H, G + 3 * H, 5 * H, U_fl, H, DX, 2 * H, 1.f));
        BL(gemm_rm(c->blas, false, false, (int)n, H, H, G + 4 * H, 5 * H, U_fr, H, DX + H, 2 * H, 1.f));
        scatter_dh<<<nblk(n * 2 * H), 256, 0, s>>>(DX, ints + 6 * r0, (int)n, H, pool);
    }
    if (n_leaf > 0) {
        leaf_bwd<<<nblk(n_leaf * H), 256, 0, s>>>(leaves, (int)n_leaf, H, pool, Gl);
        if (d_inputs) {
            BL(gemm_rm(c->blas, false, false, (int)n_leaf, E, 3 * H, Gl, 3 * H, W_iou, E, DX, E, 0.f));
            scatter_dx<<<nblk(n_leaf * E), 256, 0, s>>>(DX, leaves, (int)n_leaf, E, d_inputs);
        }
    }
    // ---- weight gradients (L185): one GEMM per matrix over the concatenated nodes ----
    BL(gemm_rm(c->blas, true, false, 3 * H, 2 * H, (int)n_int, Gi, 5 * H, Xi, 2 * H, grads + off[1], 2 * H, 0.f));
    BL(gemm_rm(c->blas, true, false, H, H, (int)n_int, Gi + 3 * H, 5 * H, Xi, 2 * H, grads + off[2], H, 0.f));
    BL(gemm_rm(c->blas, true, false, H, H, (int)n_int, Gi + 4 * H, 5 * H, Xi + H, 2 * H, grads + off[3], H, 0.f));
    BL(gemm_rm(c->blas, true, false, 3 * H, E, (int)n_leaf, Gl, 3 * H, Xl, E, grads + off[0], E, 0.f));
    bias_grads<<<nblk(4 * H), 256, 0, s>>>(Gi, (int)n_int, Gl, (int)n_leaf, H, grads + off[5], grads + off[6]);
#undef BL
    return (int)cudaGetLastError();
}

}  // namespace vpps
