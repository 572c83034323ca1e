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
// plain FP32 GEMMs (vpps_gemm.cu FFMA2 tiles, no TF32); gathers, cells, heads, scatters and bias gradients are the
// kernels below.  Pool records and adjoint blocks follow SPEC_SCRIPT §S7 (binary leaf [h c i o u | g_i g_o
// g_u], internal [h c i o u f_l f_r | g_i g_o g_u g_fl g_fr], head [p(C) loss], adj [dh | dc]).
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
// shared logits of one head: C floats, padded to whole float4 plus one more (the unrolled dh loop reads the
// logits in vector pieces; compute-sanitizer memcheck flagged the 12-byte read past an unpadded C = 5 block)
inline size_t heads_smem(int C) { return (size_t)(((C + 3) & ~3) + 4) * sizeof(float); }

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
__global__ void int_bwd(const uint32_t* __restrict__ nodes, int n, int H, float* pool, float* __restrict__ G,
                        bool shared = false) {
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
    if (shared) {             // TD-LSTM (R-37): a child may have two parents in the level
        atomicAdd(pool + e[4] + H + j, chat * fl);
        atomicAdd(pool + e[5] + H + j, chat * fr);
    } else {
        pool[e[4] + H + j] = chat * fl;
        pool[e[5] + H + j] = chat * fr;
    }
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
// Column sums with a block per 32 columns: lane = column (coalesced 128-byte rows), the 8 warps stride the
// rows with 4 independent accumulators each, then one shared-memory pass over the 8 warp partials (a fixed
// order: deterministic).  (One serial thread per column took 0.58 ms for config 5's bias gradients.)
__device__ __forceinline__ float colsum_block(const float* __restrict__ A, int64_t ld, int rows, int c, bool ok,
                                              float (*part)[33]) {
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    float s0 = 0.f, s1 = 0.f, s2 = 0.f, s3 = 0.f;
    if (ok) {
        int r = w;
        for (; r + 24 < rows; r += 32) {
            s0 += A[(int64_t)r * ld + c];
            s1 += A[(int64_t)(r + 8) * ld + c];
            s2 += A[(int64_t)(r + 16) * ld + c];
            s3 += A[(int64_t)(r + 24) * ld + c];
        }
        for (; r < rows; r += 8) s0 += A[(int64_t)r * ld + c];
    }
    part[w][lane] = (s0 + s1) + (s2 + s3);
    __syncthreads();
    float t = 0.f;
    if (w == 0)
#pragma unroll
        for (int k = 0; k < 8; ++k) t += part[k][lane];
    __syncthreads();
    return t;                                             // valid in warp 0
}

__global__ void bias_grads(const float* __restrict__ Gi, int ni, const float* __restrict__ Gl, int nl, int H,
                           float* db_iou, float* db_f) {
    __shared__ float part[8][33];
    const int k = blockIdx.x * 32 + (threadIdx.x & 31);
    const bool ok = k < 4 * H, iou = k < 3 * H;
    // column k of [G_int | G_leaf] for the i / o / u biases, columns 3H + j and 4H + j of G_int for b_f
    const float* a1 = iou ? Gi + k : Gi + 3 * H + (k - 3 * H);
    const float* a2 = iou ? Gl + k : Gi + 4 * H + (k - 3 * H);
    const float t1 = colsum_block(a1, 5 * H, ni, 0, ok, part);
    const float t2 = colsum_block(a2, iou ? 3 * H : 5 * H, iou ? nl : ni, 0, ok, part);
    if (threadIdx.x < 32 && ok) {
        if (iou) db_iou[k] = t1 + t2;
        else db_f[k - 3 * H] = t1 + t2;
    }
}

// ---- BiLSTM tagger (M2): time steps of the two directions as levels ----
__global__ void tg_gather_x(const float* __restrict__ inputs, const uint32_t* __restrict__ tok, int T, int E,
                            float* __restrict__ X) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x, q = E / 4;
    if (i >= (int64_t)T * q) return;
    const int r = (int)(i / q), c = (int)(i % q) * 4;
    *reinterpret_cast<float4*>(X + (int64_t)r * E + c) = __ldg(reinterpret_cast<const float4*>(inputs + (int64_t)tok[r] * E + c));
}

// rows of h_prev for the positions of one step: HH[pos + dp][d H .. d H + H)
__global__ void tg_gather_hprev(const float* __restrict__ HH, const uint32_t* __restrict__ pos, int n, int dp, int d,
                                int H, int HW, float* __restrict__ Hp) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    Hp[t] = HH[(int64_t)((int)pos[r] + dp) * HW + d * H + j];
}

// LSTM step (M1, gates i f o g): a = P[pos] + Zs[r] (recurrent, absent at t = 0) + b
__global__ void tg_cell(const float* __restrict__ P, const float* __restrict__ Zs, const float* __restrict__ b,
                        const uint32_t* __restrict__ pos, int n, int dp, bool first, int d, int H, int HW, float* HH,
                        float* Cd, float* Gd, float* HS) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    const int64_t p = pos[r];
    const float* pr = P + p * 4 * H;
    float a[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) a[k] = pr[k * H + j] + b[k * H + j] + (first ? 0.f : Zs[(int64_t)r * 4 * H + k * H + j]);
    const float i = sigm(a[0]), f = sigm(a[1]), o = sigm(a[2]), g = tanhf(a[3]);
    const float cp = first ? 0.f : Cd[(p + dp) * H + j];
    const float c = f * cp + i * g;
    const float h = o * tanhf(c);
    HH[p * HW + d * H + j] = h;
    HS[t] = h;                        // step-major copy: the next step's recurrent product reads it in place
    Cd[p * H + j] = c;
    float* gr = Gd + p * 4 * H;
    gr[j] = i; gr[H + j] = f; gr[2 * H + j] = o; gr[3 * H + j] = g;
}

// m = tanh(A + b_mlp) in place
__global__ void tg_tanh_bias(float* A, const float* __restrict__ b, int64_t n, int M) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t < n) A[t] = tanhf(A[t] + b[t % M]);
}

// softmax-NLL head per position (warp per position, any C): labelled positions add their NLL to the loss
// (L205) and get dZ = p - onehot(y); unlabelled positions get dZ = 0
__global__ void tg_softmax(const float* __restrict__ Z, const float* __restrict__ b_tag, const uint32_t* __restrict__ lab,
                           int T, int C, float* dZ, float* loss) {
    const int w = (int)(((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5), lane = threadIdx.x & 31;
    if (w >= T) return;
    const int y = (int)lab[w];
    const float* z = Z + (int64_t)w * C;
    float* dz = dZ + (int64_t)w * C;
    if (y < 0) { for (int c = lane; c < C; c += 32) dz[c] = 0.f; return; }
    float m = -INFINITY;
    for (int c = lane; c < C; c += 32) m = fmaxf(m, z[c] + b_tag[c]);
    m = warp_max(m);
    float se = 0.f;
    for (int c = lane; c < C; c += 32) se += expf(z[c] + b_tag[c] - m);
    const float lse = m + logf(warp_sum(se));
    for (int c = lane; c < C; c += 32) dz[c] = expf(z[c] + b_tag[c] - lse) - (c == y ? 1.f : 0.f);
    if (lane == 0) atomicAdd(loss, lse - (z[y] + b_tag[y]));
}

// dA = dM (1 - m^2) in place
__global__ void tg_dtanh(float* dM, const float* __restrict__ Mm, int64_t n) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t < n) dM[t] *= 1.f - Mm[t] * Mm[t];
}

// LSTM step backward (c.2b M1): dh = dHH[pos] (head) + dHr[pos] (from the next step), dc = dCr[pos];
// γ -> Gam[pos] and the step buffer Gs[r]; dc_prev -> dCr[pos + dp]
__global__ void tg_cell_bwd(const uint32_t* __restrict__ pos, int n, int dp, bool first, int d, int H, int HW,
                            const float* __restrict__ dHH, const float* __restrict__ DhN, int n_next, float* dCr,
                            const float* __restrict__ Cd, const float* __restrict__ Gd, float* Gam, float* Gs) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    const int64_t p = pos[r];
    // recurrent dh: row r of the successor step's Γ Uᵀ block (the successor step has n_next <= n rows)
    const float dh = dHH[p * HW + d * H + j] + (r < n_next ? DhN[t] : 0.f), dc = dCr[p * H + j];
    const float* gr = Gd + p * 4 * H;
    const float i = gr[j], f = gr[H + j], o = gr[2 * H + j], g = gr[3 * H + j];
    const float c = Cd[p * H + j], cp = first ? 0.f : Cd[(p + dp) * H + j];
    const float tc = tanhf(c);
    const float chat = dc + dh * o * (1.f - tc * tc);
    const float gam[4] = {chat * g * i * (1.f - i), chat * cp * f * (1.f - f), dh * tc * o * (1.f - o),
                          chat * i * (1.f - g * g)};
#pragma unroll
    for (int k = 0; k < 4; ++k) { Gam[p * 4 * H + k * H + j] = gam[k]; Gs[(int64_t)r * 4 * H + k * H + j] = gam[k]; }
    if (!first) dCr[(p + dp) * H + j] = chat * f;
}

// dHr[pos + dp] = Dh[r] (the step's recurrent dh contribution to its predecessor)
__global__ void tg_scatter_dh(const float* __restrict__ Dh, const uint32_t* __restrict__ pos, int n, int dp, int H, float* dHr) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    dHr[((int64_t)pos[r] + dp) * H + j] = Dh[t];
}

// Hp_all[p] = h of p's predecessor in direction d (zeros at the chain start), for dU = Γᵀ Hp_all
__global__ void tg_hprev_all(const float* __restrict__ HH, const uint32_t* __restrict__ pos, int n, int dp, int d,
                             int H, int HW, float* Hp) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    Hp[(int64_t)pos[r] * H + j] = HH[((int64_t)pos[r] + dp) * HW + d * H + j];
}

__global__ void tg_scatter_dx(const float* __restrict__ DX, const uint32_t* __restrict__ tok, int T, int E, float* dX) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)T * E) return;
    const uint32_t k = tok[t / E];
    if (k != NONE) atomicAdd(dX + (int64_t)k * E + t % E, DX[t]);   // (BiLSTMwChar's rare words: no table row)
}

// ---- BiLSTMwChar (M9, reading R-38) ----
// word input rows: the table row of a frequent word, [h→ at the last character; h← at the first character]
// of the character BiLSTM (HHc [Tc][2 Hc]) for a rare word
__global__ void wc_gather_x(const float* __restrict__ inputs, const uint32_t* __restrict__ tok,
                            const uint32_t* __restrict__ rare, const uint32_t* __restrict__ rlist,
                            const float* __restrict__ HHc, int T, int E, float* __restrict__ X) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= (int64_t)T * E) return;
    const int p = (int)(i / E), j = (int)(i % E), Hc = E / 2;
    const uint32_t k = tok[p];
    float v;
    if (k != NONE) {
        v = __ldg(inputs + (int64_t)k * E + j);
    } else {
        const uint32_t* e = rlist + 3 * rare[p];
        const int64_t q = j < Hc ? (int64_t)e[1] + e[2] - 1 : (int64_t)e[1];   // last / first character
        v = HHc[q * E + j];
    }
    X[i] = v;
}
// dh seeds of the character chains: a rare word's dX row enters at the forward direction's last character
// (columns 0 .. Hc) and at the backward direction's first character (Hc .. 2 Hc); dHHc zeroed before
__global__ void wc_seed(const float* __restrict__ DX, const uint32_t* __restrict__ rlist, int R, int E,
                        float* __restrict__ dHHc) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= (int64_t)R * E) return;
    const int r = (int)(i / E), j = (int)(i % E), Hc = E / 2;
    const uint32_t* e = rlist + 3 * r;
    const int64_t q = j < Hc ? (int64_t)e[1] + e[2] - 1 : (int64_t)e[1];
    dHHc[q * E + j] = DX[(int64_t)e[0] * E + j];
}
// h_{t-1} of every character position in direction d (0 at a spelling's start in that direction)
__global__ void wc_hprev(const float* __restrict__ HHc, const uint32_t* __restrict__ cword,
                         const uint32_t* __restrict__ rlist, int Tc, int Hc, int d, float* __restrict__ Hp) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= (int64_t)Tc * Hc) return;
    const int q = (int)(i / Hc), j = (int)(i % Hc);
    const uint32_t* e = rlist + 3 * cword[q];
    const int k = q - (int)e[1];                       // index inside the spelling
    const bool has = d == 0 ? k > 0 : k + 1 < (int)e[2];
    Hp[i] = has ? HHc[(int64_t)(d == 0 ? q - 1 : q + 1) * 2 * Hc + d * Hc + j] : 0.f;
}


// ---- GRU chains (M5, reading R-34): gates (r, z, n); a_x = W x + b_i (Px = X Wᵀ over all positions),
//      a_h = U h_prev + b_h (Zs = H_prev Uᵀ per step); the reset gate multiplies a_h[n] ----
// forward step: Gd[p] = (r, z, n, a_h[n]) for the backward
__global__ void gru_cell(const float* __restrict__ Px, const float* __restrict__ Zs, const float* __restrict__ b_i,
                         const float* __restrict__ b_h, const uint32_t* __restrict__ pos, int n, int dp, bool first,
                         int H, float* HH, float* Gd, float* HS) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    const int64_t p = pos[r];
    const float* px = Px + p * 3 * H;
    const float* zs = Zs + (int64_t)r * 3 * H;
    const float ahr = b_h[j] + (first ? 0.f : zs[j]);
    const float ahz = b_h[H + j] + (first ? 0.f : zs[H + j]);
    const float ahn = b_h[2 * H + j] + (first ? 0.f : zs[2 * H + j]);
    const float rg = sigm(px[j] + b_i[j] + ahr);
    const float zg = sigm(px[H + j] + b_i[H + j] + ahz);
    const float ng = tanhf(px[2 * H + j] + b_i[2 * H + j] + rg * ahn);
    const float hp = first ? 0.f : HH[(p + dp) * H + j];
    const float h = (1.f - zg) * ng + zg * hp;
    HH[p * H + j] = h;
    HS[t] = h;                        // step-major copy for the next step's recurrent product
    float* g = Gd + p * 4 * H;
    g[j] = rg; g[H + j] = zg; g[2 * H + j] = ng; g[3 * H + j] = ahn;
}

// backward step: dh = dHH[p] (head) + dHr[p] (successor); γ_x -> Gx[p], γ_h -> Gh[p] and the step buffer
// Gs[r]; the direct term dh ⊙ z of dh_prev -> Ez[r]
__global__ void gru_cell_bwd(const uint32_t* __restrict__ pos, int n, int dp, bool first, int H,
                             const float* __restrict__ dHH, const float* __restrict__ DhN,
                             const float* __restrict__ EzN, int n_next,
                             const float* __restrict__ HH, const float* __restrict__ Gd, float* Gx, float* Gh,
                             float* Gs, float* Ez) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    const int64_t p = pos[r];
    // recurrent dh from the successor step's row r: Γ_h U + dh ⊙ z of that step
    const float dh = dHH[p * H + j] + (r < n_next ? DhN[t] + EzN[t] : 0.f);
    const float* g = Gd + p * 4 * H;
    const float rg = g[j], zg = g[H + j], ng = g[2 * H + j], ahn = g[3 * H + j];
    const float hp = first ? 0.f : HH[(p + dp) * H + j];
    const float dan = dh * (1.f - zg) * (1.f - ng * ng);
    const float dar = dan * ahn * rg * (1.f - rg);
    const float daz = dh * (hp - ng) * zg * (1.f - zg);
    float* gx = Gx + p * 3 * H;
    float* gh = Gh + p * 3 * H;
    float* gs = Gs + (int64_t)r * 3 * H;
    gx[j] = dar; gx[H + j] = daz; gx[2 * H + j] = dan;
    gh[j] = dar; gh[H + j] = daz; gh[2 * H + j] = dan * rg;
    gs[j] = dar; gs[H + j] = daz; gs[2 * H + j] = dan * rg;
    Ez[t] = dh * zg;
}

// dHr[pos + dp] = Dh[r] + Ez[r]: the step's dh_prev = Γ_h U + dh ⊙ z
__global__ void gru_scatter_dh(const float* __restrict__ Dh, const float* __restrict__ Ez, const uint32_t* __restrict__ pos,
                               int n, int dp, int H, float* dHr) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    dHr[((int64_t)pos[r] + dp) * H + j] = Dh[t] + Ez[t];
}


// ---- RvNN (M6, reading R-35): leaf h = tanh(W_leaf x + b_leaf), internal h = tanh(W_int [h_l; h_r] + b_int);
//      records keep h at offset 0, adjoints dh at adj + 0 ----
// h = tanh(Z + b) -> pool[rec]; rows of a node list with record offsets at nodes[stride * r]
__global__ void rv_cell(const float* __restrict__ Z, const float* __restrict__ b, const uint32_t* __restrict__ nodes,
                        int stride, int n, int H, float* pool) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    pool[nodes[(int64_t)stride * r] + j] = tanhf(Z[t] + b[j]);
}

// g = dh (1 - h²) -> G rows (dh from the adjoint block nodes[stride r + adj_word])
__global__ void rv_bwd(const uint32_t* __restrict__ nodes, int stride, int adj_word, int n, int H,
                       const float* __restrict__ pool, float* __restrict__ G) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    const uint32_t* e = nodes + (int64_t)stride * r;
    const float h = __ldcg(pool + e[0] + j), dh = __ldcg(pool + e[adj_word] + j);
    G[t] = dh * (1.f - h * h);
}


// ---- TD-RNN (M7, reading R-36): leaves copy their input row; shared children take dh from two parents ----
__global__ void td_leaf(const float* __restrict__ inputs, const uint32_t* __restrict__ leaf, int n, int H, float* pool) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    const uint32_t* e = leaf + 3 * r;
    pool[e[0] + j] = e[2] == NONE ? 0.f : __ldg(inputs + (int64_t)e[2] * H + j);
}

// children's dh += DX rows with atomics (a child may have a second parent in the same level)
__global__ void scatter_dh_shared(const float* __restrict__ DX, const uint32_t* __restrict__ nodes, int n, int H,
                                  float* pool) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * 2 * H) return;
    const int r = (int)(t / (2 * H)), c = (int)(t % (2 * H));
    const uint32_t* e = nodes + 6 * r;
    atomicAdd(c < H ? pool + e[4] + c : pool + e[5] + (c - H), DX[t]);
}

// dX[token] += dh of each leaf (its adjoint block)
__global__ void td_leaf_dx(const uint32_t* __restrict__ leaf, int n, int H, const float* __restrict__ pool, float* dX) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= (int64_t)n * H) return;
    const int r = (int)(t / H), j = (int)(t % H);
    const uint32_t* e = leaf + 3 * r;
    if (e[2] != NONE) atomicAdd(dX + (int64_t)e[2] * H + j, __ldcg(pool + e[1] + j));
}

// out[y][c] = Σ_{r in row slice y} A[r][c]: one 256-thread block per 32 columns (colsum_grid) and per row
// slice (gridDim.y slices; with one slice, out[c] = the whole column sum)
__global__ void colsum(const float* __restrict__ A, int rows, int cols, float* out) {
    __shared__ float part[8][33];
    const int per = (rows + (int)gridDim.y - 1) / (int)gridDim.y, r0 = (int)blockIdx.y * per;
    const int nr = max(0, min(rows - r0, per));
    const int c = blockIdx.x * 32 + (threadIdx.x & 31);
    const float t = colsum_block(A + (int64_t)r0 * cols, cols, nr, c, c < cols, part);
    if (threadIdx.x < 32 && c < cols) out[(int64_t)blockIdx.y * cols + c] = t;
}
inline unsigned colsum_grid(int cols) { return (unsigned)((cols + 31) / 32); }

}  // namespace lv
}  // namespace dev

// ---- host orchestration ------------------------------------------------------------------------

// Row-major C[M x N] = op(A) op(B) + beta C (A: M x K, or K x M when ta; B: K x N, or N x K when tb): the
// hand-written FFMA2 tiles of vpps_gemm.cu, on the stream of the chain / level being computed
static cudaError_t gemm_rm(cudaStream_t h, bool ta, bool tb, int M, int N, int K, const float* A, int lda,
                           const float* B, int ldb, float* C, int ldc, float beta) {
    return gemm_f32(h, ta, tb, M, N, K, A, lda, B, ldb, C, ldc, beta);
}

struct LevelBufs {
    float *X_leaf = nullptr, *X_int = nullptr, *Z = nullptr, *G_int = nullptr, *G_leaf = nullptr, *DX = nullptr;
    int64_t cap_leaf = 0, cap_int = 0;
};

// work buffers grow geometrically through the model's device allocator (stream-ordered: no device sync)
static bool grow_buf(const DevAlloc* a, cudaStream_t s, float** p, int64_t* cap, int64_t need) {
    if (need <= *cap) return true;
    a->put(*p, s);
    *p = nullptr;
    *cap = 0;
    const int64_t c = need + need / 4 + 1024;
    *p = static_cast<float*>(a->get((size_t)c * sizeof(float), s));
    if (!*p) return false;
    *cap = c;
    return true;
}
#define grow(...) grow_buf(&c->alloc, s, __VA_ARGS__)


struct TaggerBufs {
    float *X = nullptr, *Pf = nullptr, *Pb = nullptr, *HH = nullptr, *Cf = nullptr, *Cb = nullptr, *Gf = nullptr,
          *Gb = nullptr, *Hp = nullptr, *Zs = nullptr, *Mm = nullptr, *Z = nullptr, *dZ = nullptr, *dM = nullptr,
          *dHH = nullptr, *dHf = nullptr, *dHb = nullptr, *dCf = nullptr, *dCb = nullptr, *Gamf = nullptr,
          *Gamb = nullptr, *Gs = nullptr, *Dh = nullptr, *DX = nullptr;
    float *Hp2 = nullptr, *Zs2 = nullptr, *Gs2 = nullptr, *Dh2 = nullptr;   // second direction's step buffers
    float *HS0 = nullptr, *HS1 = nullptr, *DhB0 = nullptr, *DhB1 = nullptr, *EzB = nullptr;   // step-major h, 2nd Dh
    int64_t cap[24] = {0};
    int64_t cap2[4] = {0};
    int64_t cap3[5] = {0};
};

struct CharBufs {
    float *Xc = nullptr, *Pf = nullptr, *Pb = nullptr, *HH = nullptr, *Cf = nullptr, *Cb = nullptr, *Gf = nullptr,
          *Gb = nullptr, *dHH = nullptr, *Gamf = nullptr, *Gamb = nullptr, *Hp = nullptr, *DX = nullptr;
    int64_t cap[13] = {0};
};

struct LevelCtx {
    DevAlloc alloc;
    cudaStream_t st = nullptr;         // stream of the pass in progress (the products run on it)
    // BiLSTM tagger: the backward-direction chain runs on a second stream, joined by events — the two
    // directions are independent until the head
    cudaStream_t s2 = nullptr;
    cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    LevelBufs b;
    TaggerBufs tg;
    // BiLSTMwChar's character BiLSTM: X_c, P_f, P_b, HH (both directions), C_f, C_b, G_f, G_b, dHH, Γ_f, Γ_b,
    // H_prev, DX_c
    CharBufs ch;
    // register-resident chain recurrence (vpps_chain.cu): tagged slots, zeroed when (re)allocated; pass tag
    float *hx = nullptr, *part = nullptr;
    int64_t cap_hx = 0, cap_part = 0;
    uint32_t epoch = 0;
    int64_t cap_X_leaf = 0, cap_X_int = 0, cap_Z = 0, cap_G_int = 0, cap_G_leaf = 0, cap_DX = 0;
    float* cs = nullptr;               // column-sum partials (row slices), on the pass stream only
    int64_t cap_cs = 0;
};

void* level_ctx_create(const DevAlloc* alloc) {
    LevelCtx* c = new LevelCtx;
    c->alloc = *alloc;
    if (cudaStreamCreateWithFlags(&c->s2, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming) != cudaSuccess) {
        delete c;
        return nullptr;
    }
    return c;
}

// out[c] = Σ_r A[r][c] (bias gradients): tall inputs in up to 16 row slices (two launches, a fixed order:
// deterministic), so more than cols / 32 blocks share the reads
static cudaError_t colsum_run(LevelCtx* c, cudaStream_t s, const float* A, int rows, int cols, float* out) {
    using namespace dev::lv;
    const int rs = rows > 1024 ? std::min(16, (rows + 511) / 512) : 1;
    if (rs == 1) {
        colsum<<<dim3(colsum_grid(cols), 1), 256, 0, s>>>(A, rows, cols, out);
        return cudaGetLastError();
    }
    if (!grow_buf(&c->alloc, s, &c->cs, &c->cap_cs, (int64_t)rs * cols)) return cudaErrorMemoryAllocation;
    colsum<<<dim3(colsum_grid(cols), rs), 256, 0, s>>>(A, rows, cols, c->cs);
    colsum<<<dim3(colsum_grid(cols), 1), 256, 0, s>>>(c->cs, rs, cols, out);
    return cudaGetLastError();
}

void level_ctx_destroy(void* p) {
    LevelCtx* c = static_cast<LevelCtx*>(p);
    if (!c) return;
    if (c->s2) cudaStreamDestroy(c->s2);
    if (c->ev_fork) cudaEventDestroy(c->ev_fork);
    if (c->ev_join) cudaEventDestroy(c->ev_join);
    float* bufs[] = {c->b.X_leaf, c->b.X_int, c->b.Z, c->b.G_int, c->b.G_leaf, c->b.DX};
    for (float* q : bufs) c->alloc.put(q, nullptr);
    TaggerBufs& t = c->tg;
    float* tbufs[] = {t.X, t.Pf, t.Pb, t.HH, t.Cf, t.Cb, t.Gf, t.Gb, t.Hp, t.Zs, t.Mm, t.Z, t.dZ, t.dM, t.dHH, t.dHf,
                      t.dHb, t.dCf, t.dCb, t.Gamf, t.Gamb, t.Gs, t.Dh, t.DX, t.Hp2, t.Zs2, t.Gs2, t.Dh2,
                      t.HS0, t.HS1, t.DhB0, t.DhB1, t.EzB};
    for (float* q : tbufs) c->alloc.put(q, nullptr);
    c->alloc.put(c->hx, nullptr);
    c->alloc.put(c->part, nullptr);
    CharBufs& cb = c->ch;
    float* cbufs[] = {cb.Xc, cb.Pf, cb.Pb, cb.HH, cb.Cf, cb.Cb, cb.Gf, cb.Gb, cb.dHH, cb.Gamf, cb.Gamb, cb.Hp, cb.DX};
    for (float* q : cbufs) c->alloc.put(q, nullptr);
    delete c;
}

static inline unsigned nblk(int64_t n, int t = 256) { return (unsigned)((n + t - 1) / t); }

// One forward + backward pass (+ dW, bias and head gradients into grads, which the caller zeroed; dX into
// d_inputs, zeroed by the caller).  Returns a CUDA error code (0 = ok).
int level_pass(void* ctx_, const float* params, const int64_t* off, float* grads, float* pool, const float* inputs,
               float* d_inputs, const uint32_t* d_blob, int64_t lv_int, int64_t lv_leaf, int64_t lv_head,
               const int32_t* lv_start, int32_t L, int64_t n_int, int64_t n_leaf, int64_t n_head, int32_t H,
               int32_t E, int32_t C, int64_t loss_word, cudaStream_t s, bool shared) {
    // shared: TD-LSTM DAGs (R-37) — children's dh and dc accumulate atomically (two parents per level)
    using namespace dev::lv;
    LevelCtx* c = static_cast<LevelCtx*>(ctx_);
    c->st = s;
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
    cudaError_t st = cudaSuccess;
#define BL(call) do { st = (call); if (st != cudaSuccess) return 1000 + (int)st; } while (0)
    // ---- forward: leaves (level 0) as one GEMM, then every internal level ----
    if (n_leaf > 0) {
        gather_leaf<<<nblk(n_leaf * (E / 4)), 256, 0, s>>>(inputs, leaves, (int)n_leaf, E, Xl);
        BL(gemm_rm(c->st, false, true, (int)n_leaf, 3 * H, E, Xl, E, W_iou, E, Z, 3 * H, 0.f));
        leaf_cell<<<nblk(n_leaf * H), 256, 0, s>>>(Z, b_iou, leaves, (int)n_leaf, H, pool);
    }
    for (int32_t l = 1; l <= L; ++l) {
        const int64_t r0 = lv_start[l], n = lv_start[l + 1] - r0;
        if (n <= 0) continue;
        float* X = Xi + r0 * 2 * H;
        gather_int<<<nblk(n * (2 * H / 4)), 256, 0, s>>>(pool, ints + 6 * r0, (int)n, H, X);
        BL(gemm_rm(c->st, false, true, (int)n, 3 * H, 2 * H, X, 2 * H, U_iou, 2 * H, Z, 5 * H, 0.f));
        BL(gemm_rm(c->st, false, true, (int)n, H, H, X, 2 * H, U_fl, H, Z + 3 * H, 5 * H, 0.f));
        BL(gemm_rm(c->st, false, true, (int)n, H, H, X + H, 2 * H, U_fr, H, Z + 4 * H, 5 * H, 0.f));
        int_cell<<<nblk(n * H), 256, 0, s>>>(Z, b_iou, b_f, ints + 6 * r0, (int)n, H, pool);
    }
    // ---- loss heads: forward and backward (they feed nothing forward) ----
    if (n_head > 0)
        heads<<<(unsigned)n_head, 256, heads_smem(C), s>>>(W_out, b_out, hl, H, C, pool, loss_word, grads + off[4],
                                                             grads + off[7]);
    // ---- backward: internal levels L .. 1, then the leaves ----
    for (int32_t l = L; l >= 1; --l) {
        const int64_t r0 = lv_start[l], n = lv_start[l + 1] - r0;
        if (n <= 0) continue;
        float* G = Gi + r0 * 5 * H;
        int_bwd<<<nblk(n * H), 256, 0, s>>>(ints + 6 * r0, (int)n, H, pool, G, shared);
        // [dh_l; dh_r] = U_iouᵀ g_iou, dh_l += U_flᵀ g_fl, dh_r += U_frᵀ g_fr
        BL(gemm_rm(c->st, false, false, (int)n, 2 * H, 3 * H, G, 5 * H, U_iou, 2 * H, DX, 2 * H, 0.f));
        BL(gemm_rm(c->st, false, false, (int)n, H, H, G + 3 * H, 5 * H, U_fl, H, DX, 2 * H, 1.f));
        BL(gemm_rm(c->st, false, false, (int)n, H, H, G + 4 * H, 5 * H, U_fr, H, DX + H, 2 * H, 1.f));
        if (shared) scatter_dh_shared<<<nblk(n * 2 * H), 256, 0, s>>>(DX, ints + 6 * r0, (int)n, H, pool);
        else scatter_dh<<<nblk(n * 2 * H), 256, 0, s>>>(DX, ints + 6 * r0, (int)n, H, pool);
    }
    if (n_leaf > 0) {
        leaf_bwd<<<nblk(n_leaf * H), 256, 0, s>>>(leaves, (int)n_leaf, H, pool, Gl);
        if (d_inputs) {
            BL(gemm_rm(c->st, false, false, (int)n_leaf, E, 3 * H, Gl, 3 * H, W_iou, E, DX, E, 0.f));
            scatter_dx<<<nblk(n_leaf * E), 256, 0, s>>>(DX, leaves, (int)n_leaf, E, d_inputs);
        }
    }
    // ---- weight gradients (L185): one GEMM per matrix over the concatenated nodes ----
    BL(gemm_rm(c->st, true, false, 3 * H, 2 * H, (int)n_int, Gi, 5 * H, Xi, 2 * H, grads + off[1], 2 * H, 0.f));
    BL(gemm_rm(c->st, true, false, H, H, (int)n_int, Gi + 3 * H, 5 * H, Xi, 2 * H, grads + off[2], H, 0.f));
    BL(gemm_rm(c->st, true, false, H, H, (int)n_int, Gi + 4 * H, 5 * H, Xi + H, 2 * H, grads + off[3], H, 0.f));
    BL(gemm_rm(c->st, true, false, 3 * H, E, (int)n_leaf, Gl, 3 * H, Xl, E, grads + off[0], E, 0.f));
    bias_grads<<<colsum_grid(4 * H), 256, 0, s>>>(Gi, (int)n_int, Gl, (int)n_leaf, H, grads + off[5], grads + off[6]);
#undef BL
    return (int)cudaGetLastError();
}


int tagger_pass(void* ctx_, const float* params, const int64_t* off, float* grads, float* pool, const float* inputs,
                float* d_inputs, const uint32_t* d_blob, int64_t tg_tok, int64_t tg_lab, int64_t tg_fpos,
                int64_t tg_bpos, const int32_t* start, int32_t maxlen, int64_t T, int32_t H, int32_t E, int32_t C,
                int32_t Mw, int32_t dirs, int64_t loss_word, cudaStream_t s, const uint32_t* chain_table,
                int32_t chain_g, const CharRows* cr) {
    // off: parameter offsets (Wf, Uf, Wb, Ub, W_mlp, W_tag, bf, bb, b_mlp, b_tag); dirs = 1 is the LSTM LM
    // (M1: W, U, -, -, -, W_out, b, -, -, b_out; the head reads h directly), Mw = 0 without the MLP
    using namespace dev::lv;
    const int HW = dirs * H;
    const bool has_mlp = Mw > 0;
    LevelCtx* c = static_cast<LevelCtx*>(ctx_);
    TaggerBufs& tb = c->tg;
    c->st = s;
    const int64_t Tn = std::max<int64_t>(T, 1);
    float** bufs[24] = {&tb.X, &tb.Pf, &tb.Pb, &tb.HH, &tb.Cf, &tb.Cb, &tb.Gf, &tb.Gb, &tb.Hp, &tb.Zs, &tb.Mm, &tb.Z,
                        &tb.dZ, &tb.dM, &tb.dHH, &tb.dHf, &tb.dHb, &tb.dCf, &tb.dCb, &tb.Gamf, &tb.Gamb, &tb.Gs, &tb.Dh,
                        &tb.DX};
    const int64_t Kh = has_mlp ? Mw : HW;         // width of the head's input
    const int64_t need[24] = {Tn * E, Tn * 4 * H, Tn * 4 * H, Tn * HW, Tn * H, Tn * H, Tn * 4 * H, Tn * 4 * H,
                              Tn * H, Tn * 4 * H, Tn * std::max<int64_t>(Mw, 1), Tn * C, Tn * C, Tn * Kh, Tn * HW,
                              Tn * H, Tn * H, Tn * H, Tn * H, Tn * 4 * H, Tn * 4 * H, Tn * 4 * H, Tn * H, Tn * E};
    for (int k = 0; k < 24; ++k)
        if (!grow(bufs[k], &tb.cap[k], need[k])) return (int)cudaErrorMemoryAllocation;
    {
        float** b3[5] = {&tb.HS0, &tb.HS1, &tb.DhB0, &tb.DhB1, &tb.EzB};
        const int64_t n3[5] = {Tn * H, dirs > 1 ? Tn * H : 4, Tn * H, dirs > 1 ? Tn * H : 4, 4};
        for (int k = 0; k < 5; ++k)
            if (!grow(b3[k], &tb.cap3[k], n3[k])) return (int)cudaErrorMemoryAllocation;
    }
    if (dirs > 1) {
        float** b2[4] = {&tb.Hp2, &tb.Zs2, &tb.Gs2, &tb.Dh2};
        const int64_t n2[4] = {Tn * H, Tn * 4 * H, Tn * 4 * H, Tn * H};
        for (int k = 0; k < 4; ++k)
            if (!grow(b2[k], &tb.cap2[k], n2[k])) return (int)cudaErrorMemoryAllocation;
    }
    auto P_ = [&](int k) -> const float* { return off[k] >= 0 ? params + off[k] : nullptr; };
    const float *Wf = P_(0), *Uf = P_(1), *Wb = P_(2), *Ub = P_(3), *Wm = P_(4), *Wt = P_(5), *bf = P_(6),
                *bb = P_(7), *bm = P_(8), *bt = P_(9);
    const uint32_t *tok = d_blob + tg_tok, *lab = d_blob + tg_lab, *fpos = d_blob + tg_fpos, *bpos = d_blob + tg_bpos;
    cudaError_t st;
#define BL(call) do { st = (call); if (st != cudaSuccess) return 1000 + (int)st; } while (0)
    if (T == 0) return 0;
    if (cr) wc_gather_x<<<nblk(T * E), 256, 0, s>>>(inputs, tok, cr->rare, cr->rlist, cr->HHc, (int)T, E, tb.X);
    else tg_gather_x<<<nblk(T * (E / 4)), 256, 0, s>>>(inputs, tok, (int)T, E, tb.X);
    BL(gemm_rm(c->st, false, true, (int)T, 4 * H, E, tb.X, E, Wf, E, tb.Pf, 4 * H, 0.f));
    if (dirs > 1) BL(gemm_rm(c->st, false, true, (int)T, 4 * H, E, tb.X, E, Wb, E, tb.Pb, 4 * H, 0.f));
    // register-resident recurrence (vpps_chain.cu): U of each direction in the registers of a group of CTAs,
    // whole sentences per group, tagged slots between the steps — one launch for the forward steps of both
    // directions, one for the backward steps (instead of a product and a cell launch per step)
    ChainParams cp{};
    const int32_t ncl = chain_table ? chain_group_ctas(H) : 0;
    const bool chain = ncl > 0 && chain_g > 0;
    if (chain) {
        // slots: HX [T][H] and PART [T][NCL][H] 64-bit words, never cleared again (epoch tags)
        const int64_t need_hx = 2 * dirs * T * H, need_part = 2 * dirs * T * (int64_t)ncl * H;
        if (need_hx > c->cap_hx) {
            if (!grow(&c->hx, &c->cap_hx, need_hx)) return (int)cudaErrorMemoryAllocation;
            cudaMemsetAsync(c->hx, 0, (size_t)c->cap_hx * sizeof(float), s);
        }
        if (need_part > c->cap_part) {
            if (!grow(&c->part, &c->cap_part, need_part)) return (int)cudaErrorMemoryAllocation;
            cudaMemsetAsync(c->part, 0, (size_t)c->cap_part * sizeof(float), s);
        }
        if (++c->epoch == 0) c->epoch = 1;
        cp.table = chain_table;
        cp.groups_dir0 = chain_g;
        cp.HW = HW;
        cp.epoch = c->epoch;
        cp.U0 = Uf; cp.U1 = dirs > 1 ? Ub : Uf; cp.b0 = bf; cp.b1 = dirs > 1 ? bb : bf;
        cp.P0 = tb.Pf; cp.P1 = tb.Pb;
        cp.HH = tb.HH;
        cp.C0 = tb.Cf; cp.C1 = tb.Cb; cp.G0 = tb.Gf; cp.G1 = tb.Gb;
        cp.dHH = tb.dHH;
        cp.Gam0 = tb.Gamf; cp.Gam1 = tb.Gamb;
        cp.hx = reinterpret_cast<unsigned long long*>(c->hx);
        cp.part = reinterpret_cast<unsigned long long*>(c->part);
        cp.T = T;
        BL(launch_chain(cp, H, chain_g * dirs, false, s));
    }
    // forward over the time steps; the two directions are independent chains: the backward one runs on
    // the second stream (its own h_prev / recurrent-product buffers), joined before the head
    if (!chain && dirs > 1) {
        cudaEventRecord(c->ev_fork, s);
        cudaStreamWaitEvent(c->s2, c->ev_fork, 0);
    }
    for (int32_t t = 0; t < (chain ? 0 : maxlen); ++t) {
        const int32_t r0 = start[t], n = start[t + 1] - r0;
        for (int d = 0; d < dirs; ++d) {
            const uint32_t* pos = (d == 0 ? fpos : bpos) + r0;
            const int dp = d == 0 ? -1 : 1;
            const float* U = d == 0 ? Uf : Ub;
            cudaStream_t sd = d == 0 ? s : c->s2;
            cudaStream_t hd = d == 0 ? c->st : c->s2;
            float* HS = d == 0 ? tb.HS0 : tb.HS1;        // step-major h of this direction
            float* Zs = d == 0 ? tb.Zs : tb.Zs2;
            if (t > 0)   // h_prev of row r = row r of the previous step's block (longest-first step lists)
                BL(gemm_rm(hd, false, true, n, 4 * H, H, HS + (int64_t)start[t - 1] * H, H, U, H, Zs, 4 * H, 0.f));
            tg_cell<<<nblk((int64_t)n * H), 256, 0, sd>>>(d == 0 ? tb.Pf : tb.Pb, Zs, d == 0 ? bf : bb, pos, n, dp,
                                                            t == 0, d, H, HW, tb.HH, d == 0 ? tb.Cf : tb.Cb,
                                                            d == 0 ? tb.Gf : tb.Gb, HS + (int64_t)r0 * H);
        }
    }
    if (!chain && dirs > 1) {
        cudaEventRecord(c->ev_join, c->s2);
        cudaStreamWaitEvent(s, c->ev_join, 0);
    }
    // head over all positions: BiLSTM tagger m = tanh(W_mlp [h→; h←] + b_mlp) (MLP 256), then
    // z = W_tag m + b_tag; LSTM LM z = W_out h + b_out (L42); forward and backward
    const float* Hin = tb.HH;
    if (has_mlp) {
        BL(gemm_rm(c->st, false, true, (int)T, Mw, HW, tb.HH, HW, Wm, HW, tb.Mm, Mw, 0.f));
        tg_tanh_bias<<<nblk(T * Mw), 256, 0, s>>>(tb.Mm, bm, T * Mw, Mw);
        Hin = tb.Mm;
    }
    BL(gemm_rm(c->st, false, true, (int)T, C, (int)Kh, Hin, (int)Kh, Wt, (int)Kh, tb.Z, C, 0.f));
    tg_softmax<<<nblk(T * 32), 256, 0, s>>>(tb.Z, bt, lab, (int)T, C, tb.dZ, pool + loss_word);
    BL(gemm_rm(c->st, true, false, C, (int)Kh, (int)T, tb.dZ, C, Hin, (int)Kh, grads + off[5], (int)Kh, 0.f));
    BL(colsum_run(c, s, tb.dZ, (int)T, C, grads + off[9]));
    if (has_mlp) {
        BL(gemm_rm(c->st, false, false, (int)T, Mw, C, tb.dZ, C, Wt, Mw, tb.dM, Mw, 0.f));
        tg_dtanh<<<nblk(T * Mw), 256, 0, s>>>(tb.dM, tb.Mm, T * Mw);
        BL(gemm_rm(c->st, true, false, Mw, HW, (int)T, tb.dM, Mw, tb.HH, HW, grads + off[4], HW, 0.f));
        BL(colsum_run(c, s, tb.dM, (int)T, Mw, grads + off[8]));
        BL(gemm_rm(c->st, false, false, (int)T, HW, Mw, tb.dM, Mw, Wm, HW, tb.dHH, HW, 0.f));
    } else {
        BL(gemm_rm(c->st, false, false, (int)T, HW, C, tb.dZ, C, Wt, HW, tb.dHH, HW, 0.f));
    }
    // backward through both LSTMs, last step first
    if (chain) BL(launch_chain(cp, H, chain_g * dirs, true, s));
    if (!chain) {
        cudaMemsetAsync(tb.dHf, 0, T * H * sizeof(float), s);
        cudaMemsetAsync(tb.dHb, 0, T * H * sizeof(float), s);
        cudaMemsetAsync(tb.dCf, 0, T * H * sizeof(float), s);
        cudaMemsetAsync(tb.dCb, 0, T * H * sizeof(float), s);
    }
    if (!chain && dirs > 1) {
        cudaEventRecord(c->ev_fork, s);
        cudaStreamWaitEvent(c->s2, c->ev_fork, 0);
    }
    for (int32_t t = chain ? -1 : maxlen - 1; t >= 0; --t) {
        const int32_t r0 = start[t], n = start[t + 1] - r0;
        for (int d = 0; d < dirs; ++d) {
            const uint32_t* pos = (d == 0 ? fpos : bpos) + r0;
            const int dp = d == 0 ? -1 : 1;
            cudaStream_t sd = d == 0 ? s : c->s2;
            cudaStream_t hd = d == 0 ? c->st : c->s2;
            float* Gs = d == 0 ? tb.Gs : tb.Gs2;
            // Γ Uᵀ of step t goes to one buffer and is read by step t-1, whose product goes to the other
            float* DhW = (t & 1) ? (d == 0 ? tb.Dh : tb.Dh2) : (d == 0 ? tb.DhB0 : tb.DhB1);
            const float* DhR = (t & 1) ? (d == 0 ? tb.DhB0 : tb.DhB1) : (d == 0 ? tb.Dh : tb.Dh2);
            const int32_t n_next = t + 1 < maxlen ? start[t + 2] - start[t + 1] : 0;
            tg_cell_bwd<<<nblk((int64_t)n * H), 256, 0, sd>>>(pos, n, dp, t == 0, d, H, HW, tb.dHH, DhR, n_next,
                                                                d == 0 ? tb.dCf : tb.dCb, d == 0 ? tb.Cf : tb.Cb,
                                                                d == 0 ? tb.Gf : tb.Gb, d == 0 ? tb.Gamf : tb.Gamb, Gs);
            if (t > 0) BL(gemm_rm(hd, false, false, n, H, 4 * H, Gs, 4 * H, d == 0 ? Uf : Ub, H, DhW, H, 0.f));
        }
    }
    if (!chain && dirs > 1) {
        cudaEventRecord(c->ev_join, c->s2);
        cudaStreamWaitEvent(s, c->ev_join, 0);
    }
    // weight gradients: dW = Γᵀ X, dU = Γᵀ H_prev (zeros at chain starts), db = Σ Γ; dX = Γf Wf + Γb Wb
    for (int d = 0; d < dirs; ++d) {
        float* Gam = d == 0 ? tb.Gamf : tb.Gamb;
        const uint32_t* pos = d == 0 ? fpos : bpos;
        const int dp = d == 0 ? -1 : 1;
        cudaMemsetAsync(tb.Hp, 0, T * H * sizeof(float), s);
        if (maxlen > 1) {
            const int32_t n = start[maxlen] - start[1];
            tg_hprev_all<<<nblk((int64_t)n * H), 256, 0, s>>>(tb.HH, pos + start[1], n, dp, d, H, HW, tb.Hp);
        }
        BL(gemm_rm(c->st, true, false, 4 * H, E, (int)T, Gam, 4 * H, tb.X, E, grads + off[d == 0 ? 0 : 2], E, 0.f));
        BL(gemm_rm(c->st, true, false, 4 * H, H, (int)T, Gam, 4 * H, tb.Hp, H, grads + off[d == 0 ? 1 : 3], H, 0.f));
        BL(colsum_run(c, s, Gam, (int)T, 4 * H, grads + off[d == 0 ? 6 : 7]));
    }
    if (d_inputs || cr) {   // (BiLSTMwChar: the rare rows' dX seeds the character chains, cr->DX = tb.DX)
        BL(gemm_rm(c->st, false, false, (int)T, E, 4 * H, tb.Gamf, 4 * H, Wf, E, tb.DX, E, 0.f));
        if (dirs > 1) BL(gemm_rm(c->st, false, false, (int)T, E, 4 * H, tb.Gamb, 4 * H, Wb, E, tb.DX, E, 1.f));
        if (d_inputs) tg_scatter_dx<<<nblk(T * E), 256, 0, s>>>(tb.DX, tok, (int)T, E, d_inputs);
    }
#undef BL
    return (int)cudaGetLastError();
}


// GRU chains (M5) on the level-synchronous path: the LSTM LM's organisation (input projections and the
// head as dense products over all positions, one recurrent product per time step, dW / dU / dX as GEMMs)
// with the GRU cell.  off: (W, U, W_out, b_i, b_h, b_out).
int gru_pass(void* ctx_, const float* params, const int64_t* off, float* grads, float* pool, const float* inputs,
             float* d_inputs, const uint32_t* d_blob, int64_t tg_tok, int64_t tg_lab, int64_t tg_fpos,
             const int32_t* start, int32_t maxlen, int64_t T, int32_t H, int32_t E, int32_t C, int64_t loss_word,
             cudaStream_t s, const uint32_t* chain_table, int32_t chain_g) {
    using namespace dev::lv;
    LevelCtx* c = static_cast<LevelCtx*>(ctx_);
    TaggerBufs& tb = c->tg;
    c->st = s;
    const int64_t Tn = std::max<int64_t>(T, 1);
    // X, Px (Pf), HH, Gd (Gf), Hp, Zs, Z, dZ, dHH, dHr (dHf), Gx (Gamf), Gh (Gamb), Gs, Dh, Ez (Cf), DX
    float** bufs[16] = {&tb.X, &tb.Pf, &tb.HH, &tb.Gf, &tb.Hp, &tb.Zs, &tb.Z, &tb.dZ, &tb.dHH, &tb.dHf, &tb.Gamf,
                        &tb.Gamb, &tb.Gs, &tb.Dh, &tb.Cf, &tb.DX};
    int64_t* caps[16] = {&tb.cap[0], &tb.cap[1], &tb.cap[3], &tb.cap[6], &tb.cap[8], &tb.cap[9], &tb.cap[11],
                         &tb.cap[12], &tb.cap[14], &tb.cap[15], &tb.cap[19], &tb.cap[20], &tb.cap[21], &tb.cap[22],
                         &tb.cap[4], &tb.cap[23]};
    const int64_t need[16] = {Tn * E, Tn * 3 * H, Tn * H, Tn * 4 * H, Tn * H, Tn * 3 * H, Tn * C, Tn * C, Tn * H,
                              Tn * H, Tn * 3 * H, Tn * 3 * H, Tn * 3 * H, Tn * H, Tn * H, Tn * E};
    for (int k = 0; k < 16; ++k)
        if (!grow(bufs[k], caps[k], need[k])) return (int)cudaErrorMemoryAllocation;
    if (!grow(&tb.HS0, &tb.cap3[0], Tn * H) || !grow(&tb.DhB0, &tb.cap3[2], Tn * H) || !grow(&tb.EzB, &tb.cap3[4], Tn * H))
        return (int)cudaErrorMemoryAllocation;
    const float *W = params + off[0], *U = params + off[1], *Wo = params + off[2], *b_i = params + off[3],
                *b_h = params + off[4], *bo = params + off[5];
    const uint32_t *tok = d_blob + tg_tok, *lab = d_blob + tg_lab, *fpos = d_blob + tg_fpos;
    cudaError_t st;
#define BL(call) do { st = (call); if (st != cudaSuccess) return 1000 + (int)st; } while (0)
    if (T == 0) return 0;
    tg_gather_x<<<nblk(T * (E / 4)), 256, 0, s>>>(inputs, tok, (int)T, E, tb.X);
    BL(gemm_rm(c->st, false, true, (int)T, 3 * H, E, tb.X, E, W, E, tb.Pf, 3 * H, 0.f));
    // register-resident recurrence (vpps_chain.cu, GRU cell): one forward and one backward launch
    ChainParams cp{};
    const int32_t ncl = chain_table ? chain_group_ctas(H) : 0;
    const bool chain = ncl > 0 && chain_g > 0;
    if (chain) {
        const int64_t need_hx = 2 * T * H, need_part = 2 * T * (int64_t)ncl * H;
        if (need_hx > c->cap_hx) {
            if (!grow(&c->hx, &c->cap_hx, need_hx)) return (int)cudaErrorMemoryAllocation;
            cudaMemsetAsync(c->hx, 0, (size_t)c->cap_hx * sizeof(float), s);
        }
        if (need_part > c->cap_part) {
            if (!grow(&c->part, &c->cap_part, need_part)) return (int)cudaErrorMemoryAllocation;
            cudaMemsetAsync(c->part, 0, (size_t)c->cap_part * sizeof(float), s);
        }
        if (++c->epoch == 0) c->epoch = 1;
        cp.table = chain_table;
        cp.groups_dir0 = chain_g;
        cp.HW = H;
        cp.epoch = c->epoch;
        cp.U0 = U; cp.U1 = U; cp.b0 = b_i; cp.b1 = b_h;
        cp.P0 = tb.Pf; cp.P1 = tb.Pf;
        cp.HH = tb.HH;
        cp.C0 = cp.C1 = nullptr;
        cp.G0 = cp.G1 = tb.Gf;
        cp.dHH = tb.dHH;
        cp.Gam0 = tb.Gamf; cp.Gam1 = tb.Gamb;
        cp.hx = reinterpret_cast<unsigned long long*>(c->hx);
        cp.part = reinterpret_cast<unsigned long long*>(c->part);
        cp.T = T;
        BL(launch_chain(cp, H, chain_g, false, s, true));
    }
    for (int32_t t = 0; t < (chain ? 0 : maxlen); ++t) {
        const int32_t r0 = start[t], n = start[t + 1] - r0;
        const uint32_t* pos = fpos + r0;
        if (t > 0)   // h_prev of row r = row r of the previous step's block (longest-first step lists)
            BL(gemm_rm(c->st, false, true, n, 3 * H, H, tb.HS0 + (int64_t)start[t - 1] * H, H, U, H, tb.Zs, 3 * H, 0.f));
        gru_cell<<<nblk((int64_t)n * H), 256, 0, s>>>(tb.Pf, tb.Zs, b_i, b_h, pos, n, -1, t == 0, H, tb.HH, tb.Gf,
                                                       tb.HS0 + (int64_t)r0 * H);
    }
    // head on h (L42): z = W_out h + b_out, softmax-NLL on labelled positions, dW_out, db_out, dh
    BL(gemm_rm(c->st, false, true, (int)T, C, H, tb.HH, H, Wo, H, tb.Z, C, 0.f));
    tg_softmax<<<nblk(T * 32), 256, 0, s>>>(tb.Z, bo, lab, (int)T, C, tb.dZ, pool + loss_word);
    BL(gemm_rm(c->st, true, false, C, H, (int)T, tb.dZ, C, tb.HH, H, grads + off[2], H, 0.f));
    BL(colsum_run(c, s, tb.dZ, (int)T, C, grads + off[5]));
    BL(gemm_rm(c->st, false, false, (int)T, H, C, tb.dZ, C, Wo, H, tb.dHH, H, 0.f));
    if (chain) BL(launch_chain(cp, H, chain_g, true, s, true));
    else cudaMemsetAsync(tb.dHf, 0, T * H * sizeof(float), s);
    for (int32_t t = chain ? -1 : maxlen - 1; t >= 0; --t) {
        const int32_t r0 = start[t], n = start[t + 1] - r0;
        const uint32_t* pos = fpos + r0;
        // Γ_h U and dh ⊙ z of step t go to one buffer pair, read by step t-1 (row-aligned)
        float* DhW = (t & 1) ? tb.Dh : tb.DhB0;
        float* EzW = (t & 1) ? tb.Cf : tb.EzB;
        const float* DhR = (t & 1) ? tb.DhB0 : tb.Dh;
        const float* EzR = (t & 1) ? tb.EzB : tb.Cf;
        const int32_t n_next = t + 1 < maxlen ? start[t + 2] - start[t + 1] : 0;
        gru_cell_bwd<<<nblk((int64_t)n * H), 256, 0, s>>>(pos, n, -1, t == 0, H, tb.dHH, DhR, EzR, n_next, tb.HH,
                                                           tb.Gf, tb.Gamf, tb.Gamb, tb.Gs, EzW);
        if (t > 0) BL(gemm_rm(c->st, false, false, n, H, 3 * H, tb.Gs, 3 * H, U, H, DhW, H, 0.f));
    }
    // dW = Γ_xᵀ X, dU = Γ_hᵀ H_prev (zeros at chain starts), db_i = Σ Γ_x, db_h = Σ Γ_h; dX = Γ_x W
    cudaMemsetAsync(tb.Hp, 0, T * H * sizeof(float), s);
    if (maxlen > 1) {
        const int32_t n = start[maxlen] - start[1];
        tg_hprev_all<<<nblk((int64_t)n * H), 256, 0, s>>>(tb.HH, fpos + start[1], n, -1, 0, H, H, tb.Hp);
    }
    BL(gemm_rm(c->st, true, false, 3 * H, E, (int)T, tb.Gamf, 3 * H, tb.X, E, grads + off[0], E, 0.f));
    BL(gemm_rm(c->st, true, false, 3 * H, H, (int)T, tb.Gamb, 3 * H, tb.Hp, H, grads + off[1], H, 0.f));
    BL(colsum_run(c, s, tb.Gamf, (int)T, 3 * H, grads + off[3]));
    BL(colsum_run(c, s, tb.Gamb, (int)T, 3 * H, grads + off[4]));
    if (d_inputs) {
        BL(gemm_rm(c->st, false, false, (int)T, E, 3 * H, tb.Gamf, 3 * H, W, E, tb.DX, E, 0.f));
        tg_scatter_dx<<<nblk(T * E), 256, 0, s>>>(tb.DX, tok, (int)T, E, d_inputs);
    }
#undef BL
    return (int)cudaGetLastError();
}


// RvNN (M6) on the level-synchronous path: leaves as one GEMM, every internal level as one gathered product,
// dW_int / dW_leaf as one GEMM each over the concatenated nodes (L185).  off: (W_leaf, W_int, W_out,
// b_leaf, b_int, b_out).  Buffers: X_leaf [n_leaf E], X_int [n_int 2H], Z, G_int [n_int H], G_leaf, DX.
int rvnn_pass(void* ctx_, const float* params, const int64_t* off, float* grads, float* pool, const float* inputs,
              float* d_inputs, const uint32_t* d_blob, int64_t lv_int, int64_t lv_leaf, int64_t lv_head,
              const int32_t* lv_start, int32_t L, int64_t n_int, int64_t n_leaf, int64_t n_head, int32_t H,
              int32_t E, int32_t C, int64_t loss_word, cudaStream_t s) {
    using namespace dev::lv;
    LevelCtx* c = static_cast<LevelCtx*>(ctx_);
    c->st = s;
    if (!grow(&c->b.X_leaf, &c->cap_X_leaf, std::max<int64_t>(n_leaf * E, 4)) ||
        !grow(&c->b.X_int, &c->cap_X_int, std::max<int64_t>(n_int * 2 * H, 4)) ||
        !grow(&c->b.Z, &c->cap_Z, std::max<int64_t>(std::max(n_leaf, n_int) * H, 4)) ||
        !grow(&c->b.G_int, &c->cap_G_int, std::max<int64_t>(n_int * H, 4)) ||
        !grow(&c->b.G_leaf, &c->cap_G_leaf, std::max<int64_t>(n_leaf * H, 4)) ||
        !grow(&c->b.DX, &c->cap_DX, std::max<int64_t>(std::max<int64_t>(n_int * 2 * H, n_leaf * E), 4)))
        return (int)cudaErrorMemoryAllocation;
    const float *W_leaf = params + off[0], *W_int = params + off[1], *W_out = params + off[2];
    const float *b_leaf = params + off[3], *b_int = params + off[4], *b_out = params + off[5];
    const uint32_t* ints = d_blob + lv_int;      // (rec, rec_l, rec_r, adj, adj_l, adj_r) per internal node
    const uint32_t* leaves = d_blob + lv_leaf;   // (rec, adj, token) per leaf
    const uint32_t* hl = d_blob + lv_head;
    float *Xl = c->b.X_leaf, *Xi = c->b.X_int, *Z = c->b.Z, *Gi = c->b.G_int, *Gl = c->b.G_leaf, *DX = c->b.DX;
    cudaError_t st = cudaSuccess;
#define BL(call) do { st = (call); if (st != cudaSuccess) return 1000 + (int)st; } while (0)
    if (n_leaf > 0) {
        gather_leaf<<<nblk(n_leaf * (E / 4)), 256, 0, s>>>(inputs, leaves, (int)n_leaf, E, Xl);
        BL(gemm_rm(c->st, false, true, (int)n_leaf, H, E, Xl, E, W_leaf, E, Z, H, 0.f));
        rv_cell<<<nblk(n_leaf * H), 256, 0, s>>>(Z, b_leaf, leaves, 3, (int)n_leaf, H, pool);
    }
    for (int32_t l = 1; l <= L; ++l) {
        const int64_t r0 = lv_start[l], n = lv_start[l + 1] - r0;
        if (n <= 0) continue;
        float* X = Xi + r0 * 2 * H;
        gather_int<<<nblk(n * (2 * H / 4)), 256, 0, s>>>(pool, ints + 6 * r0, (int)n, H, X);
        BL(gemm_rm(c->st, false, true, (int)n, H, 2 * H, X, 2 * H, W_int, 2 * H, Z, H, 0.f));
        rv_cell<<<nblk(n * H), 256, 0, s>>>(Z, b_int, ints + 6 * r0, 6, (int)n, H, pool);
    }
    if (n_head > 0)
        heads<<<(unsigned)n_head, 256, heads_smem(C), s>>>(W_out, b_out, hl, H, C, pool, loss_word, grads + off[2],
                                                             grads + off[5]);
    for (int32_t l = L; l >= 1; --l) {
        const int64_t r0 = lv_start[l], n = lv_start[l + 1] - r0;
        if (n <= 0) continue;
        float* G = Gi + r0 * H;
        rv_bwd<<<nblk(n * H), 256, 0, s>>>(ints + 6 * r0, 6, 3, (int)n, H, pool, G);
        BL(gemm_rm(c->st, false, false, (int)n, 2 * H, H, G, H, W_int, 2 * H, DX, 2 * H, 0.f));
        scatter_dh<<<nblk(n * 2 * H), 256, 0, s>>>(DX, ints + 6 * r0, (int)n, H, pool);
    }
    if (n_leaf > 0) {
        rv_bwd<<<nblk(n_leaf * H), 256, 0, s>>>(leaves, 3, 1, (int)n_leaf, H, pool, Gl);
        if (d_inputs) {
            BL(gemm_rm(c->st, false, false, (int)n_leaf, E, H, Gl, H, W_leaf, E, DX, E, 0.f));
            scatter_dx<<<nblk(n_leaf * E), 256, 0, s>>>(DX, leaves, (int)n_leaf, E, d_inputs);
        }
        BL(gemm_rm(c->st, true, false, H, E, (int)n_leaf, Gl, H, Xl, E, grads + off[0], E, 0.f));
        BL(colsum_run(c, s, Gl, (int)n_leaf, H, grads + off[3]));
    }
    if (n_int > 0) {
        BL(gemm_rm(c->st, true, false, H, 2 * H, (int)n_int, Gi, H, Xi, 2 * H, grads + off[1], 2 * H, 0.f));
        BL(colsum_run(c, s, Gi, (int)n_int, H, grads + off[4]));
    }
#undef BL
    return (int)cudaGetLastError();
}


// TD-RNN (M7) on the level-synchronous path: level k of every sentence's pyramid as one gathered product;
// a child of two parents of the same level receives both dh contributions atomically.  off: (W, W_out, b,
// b_out).  E == H.
int tdrnn_pass(void* ctx_, const float* params, const int64_t* off, float* grads, float* pool, const float* inputs,
               float* d_inputs, const uint32_t* d_blob, int64_t lv_int, int64_t lv_leaf, int64_t lv_head,
               const int32_t* lv_start, int32_t L, int64_t n_int, int64_t n_leaf, int64_t n_head, int32_t H,
               int32_t E, int32_t C, int64_t loss_word, cudaStream_t s) {
    using namespace dev::lv;
    (void)E;
    LevelCtx* c = static_cast<LevelCtx*>(ctx_);
    c->st = s;
    if (!grow(&c->b.X_int, &c->cap_X_int, std::max<int64_t>(n_int * 2 * H, 4)) ||
        !grow(&c->b.Z, &c->cap_Z, std::max<int64_t>(n_int * H, 4)) ||
        !grow(&c->b.G_int, &c->cap_G_int, std::max<int64_t>(n_int * H, 4)) ||
        !grow(&c->b.DX, &c->cap_DX, std::max<int64_t>(n_int * 2 * H, 4)))
        return (int)cudaErrorMemoryAllocation;
    const float *W = params + off[0], *W_out = params + off[1], *b = params + off[2], *b_out = params + off[3];
    const uint32_t* ints = d_blob + lv_int;
    const uint32_t* leaves = d_blob + lv_leaf;
    const uint32_t* hl = d_blob + lv_head;
    float *Xi = c->b.X_int, *Z = c->b.Z, *Gi = c->b.G_int, *DX = c->b.DX;
    cudaError_t st = cudaSuccess;
#define BL(call) do { st = (call); if (st != cudaSuccess) return 1000 + (int)st; } while (0)
    if (n_leaf > 0) td_leaf<<<nblk(n_leaf * H), 256, 0, s>>>(inputs, leaves, (int)n_leaf, H, pool);
    for (int32_t l = 1; l <= L; ++l) {
        const int64_t r0 = lv_start[l], n = lv_start[l + 1] - r0;
        if (n <= 0) continue;
        float* X = Xi + r0 * 2 * H;
        gather_int<<<nblk(n * (2 * H / 4)), 256, 0, s>>>(pool, ints + 6 * r0, (int)n, H, X);
        BL(gemm_rm(c->st, false, true, (int)n, H, 2 * H, X, 2 * H, W, 2 * H, Z, H, 0.f));
        rv_cell<<<nblk(n * H), 256, 0, s>>>(Z, b, ints + 6 * r0, 6, (int)n, H, pool);
    }
    if (n_head > 0)
        heads<<<(unsigned)n_head, 256, heads_smem(C), s>>>(W_out, b_out, hl, H, C, pool, loss_word, grads + off[1],
                                                             grads + off[3]);
    for (int32_t l = L; l >= 1; --l) {
        const int64_t r0 = lv_start[l], n = lv_start[l + 1] - r0;
        if (n <= 0) continue;
        float* G = Gi + r0 * H;
        rv_bwd<<<nblk(n * H), 256, 0, s>>>(ints + 6 * r0, 6, 3, (int)n, H, pool, G);
        BL(gemm_rm(c->st, false, false, (int)n, 2 * H, H, G, H, W, 2 * H, DX, 2 * H, 0.f));
        scatter_dh_shared<<<nblk(n * 2 * H), 256, 0, s>>>(DX, ints + 6 * r0, (int)n, H, pool);
    }
    if (n_leaf > 0 && d_inputs) td_leaf_dx<<<nblk(n_leaf * H), 256, 0, s>>>(leaves, (int)n_leaf, H, pool, d_inputs);
    if (n_int > 0) {
        BL(gemm_rm(c->st, true, false, H, 2 * H, (int)n_int, Gi, H, Xi, 2 * H, grads + off[0], 2 * H, 0.f));
        BL(colsum_run(c, s, Gi, (int)n_int, H, grads + off[2]));
    }
#undef BL
    return (int)cudaGetLastError();
}

}  // namespace vpps

namespace vpps {

// BiLSTMwChar (M9, PAPER L267 / L281, reading R-38).  The rare words' spellings run through a character
// BiLSTM on the chain recurrence (hidden Hc = E / 2 per direction; C_emb rows as its inputs, W_c x as one
// GEMM per direction), its final states become the rare positions' input rows of the word tagger
// (tagger_pass with CharRows), and the tagger's dX rows of those positions seed dh at the final states of the
// character chains on the way back; dW / dU / db of the character LSTMs and dC_emb (scatter of Γ W_c by
// character id) as dense products.  The character passes tag their slots with their own pass counter value.
int bilstmchar_pass(void* ctx_, const float* params, const int64_t* off, float* grads, float* pool,
                    const float* inputs, float* d_inputs, const uint32_t* d_blob, int64_t tg_tok, int64_t tg_lab,
                    int64_t tg_fpos, int64_t tg_bpos, const int32_t* start, int32_t maxlen, int64_t T, int32_t H,
                    int32_t E, int32_t C, int32_t Mw, int64_t loss_word, cudaStream_t s, const uint32_t* chain_table,
                    int32_t chain_g, int64_t tc_T, int64_t tc_R, int64_t tc_tok, int64_t tc_word, int64_t tc_rare,
                    int64_t tc_list, int64_t tc_chain, int32_t chain_gc, int32_t Ec) {
    using namespace dev::lv;
    LevelCtx* c = static_cast<LevelCtx*>(ctx_);
    c->st = s;
    const int32_t Hc = E / 2;
    const int64_t Tc = tc_T, R = tc_R;
    const int64_t off10[10] = {off[0], off[1], off[2], off[3], off[4], off[5], off[11], off[12], off[13], off[14]};
    const uint32_t* ctok = d_blob + tc_tok;
    const uint32_t* cword = d_blob + tc_word;
    CharRows cr{d_blob + tc_rare, d_blob + tc_list, nullptr};
    cudaError_t st;
#define BL(call) do { st = (call); if (st != cudaSuccess) return 1000 + (int)st; } while (0)
    ChainParams cp{};
    uint32_t e_chars = 0;
    const int32_t ncl = chain_group_ctas(Hc);
    CharBufs& cb = c->ch;
    if (R > 0) {
        if (tc_chain < 0 || ncl <= 0) return (int)cudaErrorInvalidValue;
        const int64_t Tn = std::max<int64_t>(Tc, 1);
        float** bufs[13] = {&cb.Xc, &cb.Pf, &cb.Pb, &cb.HH, &cb.Cf, &cb.Cb, &cb.Gf, &cb.Gb, &cb.dHH, &cb.Gamf, &cb.Gamb,
                            &cb.Hp, &cb.DX};
        const int64_t need[13] = {Tn * Ec, Tn * 4 * Hc, Tn * 4 * Hc, Tn * E, Tn * Hc, Tn * Hc, Tn * 4 * Hc, Tn * 4 * Hc,
                                  Tn * E, Tn * 4 * Hc, Tn * 4 * Hc, Tn * Hc, Tn * Ec};
        for (int k = 0; k < 13; ++k)
            if (!grow(bufs[k], &cb.cap[k], need[k])) return (int)cudaErrorMemoryAllocation;
        const int64_t need_hx = 2 * 2 * Tc * Hc, need_part = 2 * 2 * Tc * (int64_t)ncl * Hc;
        if (need_hx > c->cap_hx) {
            if (!grow(&c->hx, &c->cap_hx, need_hx)) return (int)cudaErrorMemoryAllocation;
            cudaMemsetAsync(c->hx, 0, (size_t)c->cap_hx * sizeof(float), s);
        }
        if (need_part > c->cap_part) {
            if (!grow(&c->part, &c->cap_part, need_part)) return (int)cudaErrorMemoryAllocation;
            cudaMemsetAsync(c->part, 0, (size_t)c->cap_part * sizeof(float), s);
        }
        if (++c->epoch == 0) c->epoch = 1;
        e_chars = c->epoch;
        const float *Cemb = params + off[6], *Wcf = params + off[7], *Ucf = params + off[8], *Wcb = params + off[9],
                    *Ucb = params + off[10], *bcf = params + off[15], *bcb = params + off[16];
        // character BiLSTM forward: C_emb rows, input projections, the recurrence of both directions
        tg_gather_x<<<nblk(Tc * (Ec / 4)), 256, 0, s>>>(Cemb, ctok, (int)Tc, Ec, cb.Xc);
        BL(gemm_rm(s, false, true, (int)Tc, 4 * Hc, Ec, cb.Xc, Ec, Wcf, Ec, cb.Pf, 4 * Hc, 0.f));
        BL(gemm_rm(s, false, true, (int)Tc, 4 * Hc, Ec, cb.Xc, Ec, Wcb, Ec, cb.Pb, 4 * Hc, 0.f));
        cp.table = d_blob + tc_chain;
        cp.groups_dir0 = chain_gc;
        cp.HW = E;
        cp.epoch = e_chars;
        cp.U0 = Ucf; cp.U1 = Ucb; cp.b0 = bcf; cp.b1 = bcb;
        cp.P0 = cb.Pf; cp.P1 = cb.Pb;
        cp.HH = cb.HH;
        cp.C0 = cb.Cf; cp.C1 = cb.Cb; cp.G0 = cb.Gf; cp.G1 = cb.Gb;
        cp.dHH = cb.dHH;
        cp.Gam0 = cb.Gamf; cp.Gam1 = cb.Gamb;
        cp.hx = reinterpret_cast<unsigned long long*>(c->hx);
        cp.part = reinterpret_cast<unsigned long long*>(c->part);
        cp.T = Tc;
        BL(launch_chain(cp, Hc, 2 * chain_gc, false, s));
        cr.HHc = cb.HH;
    }
    // the word tagger over the rows [table row | character states]
    int rc = tagger_pass(ctx_, params, off10, grads, pool, inputs, d_inputs, d_blob, tg_tok, tg_lab, tg_fpos, tg_bpos,
                         start, maxlen, T, H, E, C, Mw, 2, loss_word, s, chain_table, chain_g, R > 0 ? &cr : nullptr);
    if (rc != 0 || R == 0) return rc;
    // character backward: seeds from the rare rows' dX, the recurrence, then the parameter gradients
    cudaMemsetAsync(cb.dHH, 0, (size_t)Tc * E * sizeof(float), s);
    wc_seed<<<nblk(R * E), 256, 0, s>>>(c->tg.DX, d_blob + tc_list, (int)R, E, cb.dHH);
    cp.hx = reinterpret_cast<unsigned long long*>(c->hx);       // (the word pass may have grown the slots)
    cp.part = reinterpret_cast<unsigned long long*>(c->part);
    BL(launch_chain(cp, Hc, 2 * chain_gc, true, s));
    const float *Wcf = params + off[7], *Wcb = params + off[9];
    for (int d = 0; d < 2; ++d) {
        float* Gam = d == 0 ? cb.Gamf : cb.Gamb;
        wc_hprev<<<nblk(Tc * Hc), 256, 0, s>>>(cb.HH, cword, d_blob + tc_list, (int)Tc, Hc, d, cb.Hp);
        BL(gemm_rm(s, true, false, 4 * Hc, Ec, (int)Tc, Gam, 4 * Hc, cb.Xc, Ec, grads + off[d == 0 ? 7 : 9], Ec, 0.f));
        BL(gemm_rm(s, true, false, 4 * Hc, Hc, (int)Tc, Gam, 4 * Hc, cb.Hp, Hc, grads + off[d == 0 ? 8 : 10], Hc, 0.f));
        BL(colsum_run(c, s, Gam, (int)Tc, 4 * Hc, grads + off[d == 0 ? 15 : 16]));
    }
    BL(gemm_rm(s, false, false, (int)Tc, Ec, 4 * Hc, cb.Gamf, 4 * Hc, Wcf, Ec, cb.DX, Ec, 0.f));
    BL(gemm_rm(s, false, false, (int)Tc, Ec, 4 * Hc, cb.Gamb, 4 * Hc, Wcb, Ec, cb.DX, Ec, 1.f));
    tg_scatter_dx<<<nblk(Tc * Ec), 256, 0, s>>>(cb.DX, ctok, (int)Tc, Ec, grads + off[6]);
#undef BL
    return (int)cudaGetLastError();
}

}  // namespace vpps
