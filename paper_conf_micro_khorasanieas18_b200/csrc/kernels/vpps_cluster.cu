// VPPS on thread-block clusters (sm_100a) — binary Tree-LSTM.
//
// A replica group of the partition plan (SPEC P1) is one cluster of 16 CTAs on 16 SMs: together their
// register files hold every weight matrix of the model once (weights cached in registers
// for the whole pass).  Whole graphs are assigned to clusters (SPEC S5g), so no node depends on another
// cluster and the signal/wait instructions of the script (L165) become the hardware cluster barrier
// (barrier.cluster.arrive.release / wait.acquire, ~400 cycles) instead of a grid-wide counter barrier.
// Registers cannot hold the weights and their gradients at 16 CTAs per replica, so the kernel applies
// the paper's gradient-accumulation strategy (L185, §III-C2): it records the outer-product operands
// (the gate gradients, next to the activations already in the pool) and one GEMM per weight matrix
// (vpps_dw_gemm below) forms dW = Σ g xᵀ afterwards, fused with the SGD update (L129, L197).
#include <algorithm>
#include <cstdlib>
#include "vpps_kernel.cuh"
#include "dev_common.cuh"

namespace vpps {
namespace dev {
namespace cl {

constexpr int NTH = 256;
constexpr int CHUNK = 4096;    // script words staged in shared memory (L171)
constexpr int NB = 16;         // nodes per batch: one node per lane of a unit's 16-lane group
constexpr int NC = 2;          // nodes per transposed-product chunk
constexpr int ZC = 32;         // classes per head (C <= 32)
constexpr int CINMAX = 10;
constexpr int DFW = 10;        // deferred-store entry: 3 addresses + up to 7 values
enum : uint32_t { S = 0x01, W = 0x02, LEAF_F = 0x20, LEAF_B = 0x21, INT_F = 0x22, INT_B = 0x23, HEAD_F = 0x40, HEAD_B = 0x41 };

__device__ __forceinline__ int words(uint32_t w) {
    switch (w & 0xFF) {
        case LEAF_F: return 3;
        case LEAF_B: return 4;
        case INT_F: return 4;
        case INT_B: return 7;
        case HEAD_F: return 4;
        case HEAD_B: return 5;
        default: return 1;
    }
}
__device__ __forceinline__ int n_cin(uint32_t op) {
    return op == INT_F ? 2 : op == INT_B ? 10 : op == LEAF_B ? 6 : 0;
}
// Address of cell operand k of (instruction I, unit jj); records [h c i o u (fl fr) | g...] (SPEC §S7).
template <int H>
__device__ __forceinline__ const float* cin_src(uint32_t op, const uint32_t* I, int k, int jj, const float* pool) {
    if (op == INT_F) return pool + (k == 0 ? I[2] : I[3]) + H + jj;                // c_l, c_r
    const uint32_t rec = I[1], adj = I[2];
    if (k < 2) return pool + adj + k * H + jj;                                     // dh, dc
    if (k < 8) return pool + rec + (k - 1) * H + jj;                               // c i o u (fl fr)
    return pool + (k == 8 ? I[3] : I[5]) + H + jj;                                 // c_l, c_r
}

__device__ __forceinline__ void cluster_arrive() { asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory"); }
__device__ __forceinline__ void cluster_wait() { asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory"); }
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t cluster_index() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(r));
    return r;
}

template <int H, int E>
struct CCfg {
    static constexpr int NCL = 16;                 // CTAs per cluster (= per replica)
    static constexpr int UM = H / NCL;             // hidden units per CTA
    static constexpr int TU = NTH / UM;            // threads per unit
    static_assert(H % NCL == 0 && TU == 16, "cluster kernel: 16 units per CTA, 16 threads per unit");
    using LA = Lay<E, TU>;                         // leaf bundle rows (i, o, u of W_iou) over x
    using LB = Lay<2 * H, TU>;                     // internal bundle rows (i, o, u of U_iou; f) over [h_l; h_r]
    static constexpr int KPMAX = LA::KP > LB::KP ? LA::KP : LB::KP;
    static constexpr int O_X = CHUNK;
    static constexpr int O_DXB = O_X + NB * KPMAX;
    static constexpr int O_CIN = O_DXB + UM * NC * KPMAX;
    static constexpr int O_BIAS = O_CIN + NB * UM * CINMAX;
    static constexpr int O_IPOS = O_BIAS + UM * 4;
    static constexpr int O_BST = O_IPOS + NB;
    static constexpr int O_SEGP = O_BST + 4;                 // NB x 2 pointers (8-byte aligned)
    static constexpr int O_ZS = O_SEGP + 4 * NB;
    static constexpr int O_DFW = O_ZS + NB * ZC;             // deferred stores: NB x UM entries of DFW words
    static constexpr int O_HEAD = O_DFW + NB * UM * DFW;
    static size_t smem_bytes(int32_t C) { return 4 * (size_t)(O_HEAD + 2 * C * H + 2 * C + 8); }
};

template <int H, int E>
__global__ void __launch_bounds__(NTH, 1) vpps_cl(const KParams P) {
    using T = CCfg<H, E>;
    using LA = typename T::LA;
    using LB = typename T::LB;
    constexpr int TU = T::TU, UM = T::UM, NCL = T::NCL;
    extern __shared__ __align__(16) uint32_t smw[];
    float* sm = reinterpret_cast<float*>(smw);
    uint32_t* chunk = smw;
    float* xs = sm + T::O_X;
    float* dxb = sm + T::O_DXB;
    float* cin = sm + T::O_CIN;
    float* bias = sm + T::O_BIAS;
    int* ipos = reinterpret_cast<int*>(smw + T::O_IPOS);
    int* bst = reinterpret_cast<int*>(smw + T::O_BST);
    const float** segp = reinterpret_cast<const float**>(smw + T::O_SEGP);
    float* zs = sm + T::O_ZS;
    uint32_t* dfw = smw + T::O_DFW;
    const int C = P.C;
    float* Wo = sm + T::O_HEAD;
    float* dWo = Wo + C * H;
    float* bo = dWo + C * H;
    float* dbo = bo + C;

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int lc = (int)cluster_rank(), grp = (int)cluster_index();
    const uint32_t* S_ = P.script;
    const uint32_t G = S_[0];
    const uint32_t hdr = 2 + G + 1;
    const uint32_t s0 = hdr + S_[2 + grp], s1 = hdr + S_[3 + grp];
    float* pool = P.pool;
    const int64_t* off = P.off;
    const int u = tid / TU, tu = tid % TU, gl = lane & 15;      // unit slot, thread in unit, lane in group
    const int j = lc + u * NCL;                                 // hidden unit of this thread
    const bool holds_head = (lc == H % NCL);

    // the gradient GEMM may launch now (programmatic dependent launch): its tiles wait on P.done per group
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    // ---- prologue: this CTA's slice of every weight matrix DRAM -> registers (L123, L129) ----
    // Only the recurrent matrices (U_iou, U_fl, U_fr) live in registers: the leaf level is one dense
    // GEMM over all leaves (same W_iou), done by vpps_leaf_fwd / vpps_leaf_dx around this kernel.
    float wb[4][LB::NREG];
#pragma unroll
    for (int r = 0; r < 4; ++r)
#pragma unroll
        for (int t = 0; t < LB::NT; ++t)
#pragma unroll
            for (int q = 0; q < LB::CG; ++q) {
                const int col = LB::CG * (tu + TU * t) + q;
                float v = 0.f;
                if (col < 2 * H) {
                    if (r < 3) v = __ldg(P.params + off[1] + (int64_t)(r * H + j) * (2 * H) + col);
                    else v = __ldg(P.params + (col < H ? off[2] + (int64_t)j * H + col : off[3] + (int64_t)j * H + col - H));
                }
                wb[r][t * LB::CG + q] = v;
            }
    if (tid < UM * 4) {
        const int uu = tid / 4, k = tid % 4, jj = lc + uu * NCL;
        bias[tid] = k < 3 ? __ldg(P.params + off[5] + k * H + jj) : __ldg(P.params + off[6] + jj);
    }
    if (holds_head) {
        for (int i = tid; i < C * H; i += NTH) { Wo[i] = __ldg(P.params + off[4] + i); dWo[i] = 0.f; }
        for (int i = tid; i < C; i += NTH) { bo[i] = __ldg(P.params + off[7] + i); dbo[i] = 0.f; }
    }
    float dbacc[4] = {0.f, 0.f, 0.f, 0.f};       // bias gradients of (unit u) over the nodes of slot gl
    uint64_t* prof = P.prof ? P.prof + (int64_t)blockIdx.x * P.prof_stride : nullptr;
    // section clocks (trace only): 0 decode, 1 staging, 2 forward, 3 cell-bwd, 4 transposed, 5 heads,
    // 6 signal, 7 wait, 8/9 other
    uint64_t sec[10] = {0, 0, 0, 0, 0, 0, 0, 0, 0, 0};
    uint64_t sec_last = 0;
    int sec_cur = 9;
    auto mark = [&](int k) {
        if (prof && tid == 0) {
            const uint64_t now = clock64(), d = now - sec_last;
            switch (sec_cur) {
                case 0: sec[0] += d; break;
                case 1: sec[1] += d; break;
                case 2: sec[2] += d; break;
                case 3: sec[3] += d; break;
                case 4: sec[4] += d; break;
                case 5: sec[5] += d; break;
                case 6: sec[6] += d; break;
                case 7: sec[7] += d; break;
                case 8: sec[8] += d; break;
                default: sec[9] += d; break;
            }
            sec_cur = k;
            sec_last = now;
        }
    };
    // the leaf level (vpps_leaf_fwd, the preceding grid) must be complete and visible from here on; the
    // weight loads above overlapped its tail
    asm volatile("griddepcontrol.wait;" ::: "memory");
    __syncthreads();
    if (prof && tid == 0) { prof[0] = gtimer(); sec_last = clock64(); }

    // ---- script interpretation (L171-177) ----
    uint32_t cbase = s0;
    auto refill = [&](uint32_t from) {
        __syncthreads();
        constexpr int PER = CHUNK / NTH;
        uint32_t w[PER];
#pragma unroll
        for (int i = 0; i < PER; ++i) {
            const uint32_t k = tid + i * NTH;
            w[i] = from + k < s1 ? __ldg(S_ + from + k) : 0u;
        }
#pragma unroll
        for (int i = 0; i < PER; ++i) chunk[tid + i * NTH] = w[i];
        __syncthreads();
        cbase = from;
    };
    if (s0 < s1) refill(s0);
    bool pending = false;
    bool predecoded = false;
    int n_dfr = 0;                 // deferred record stores of the last batch (entries n * UM + u)
    uint32_t dfr_op = 0;
    uint32_t pos = s0;
    // Deferred stores: the record fields no other CTA reads during the pass (c, gates, gate gradients,
    // dc of the children) are parked in shared memory and written after the next barrier arrive, so the
    // arrive's release only waits for the cross-CTA data (h, dh) and the writes drain during the wait.
    auto flush = [&]() {
        if (n_dfr == 0) return;
        __syncthreads();
        if (tid < n_dfr) {
            const uint32_t* e = dfw + tid * DFW;
            const float* v = reinterpret_cast<const float*>(e + 3);
            const int jj = lc + (tid % UM) * NCL;
            if (dfr_op == INT_F) {
#pragma unroll
                for (int k = 0; k < 6; ++k) pool[e[0] + (k + 1) * H + jj] = v[k];          // c i o u fl fr
            } else if (dfr_op == INT_B) {
#pragma unroll
                for (int k = 0; k < 5; ++k) pool[e[0] + (7 + k) * H + jj] = v[k];          // g_i g_o g_u g_fl g_fr
                pool[e[1] + H + jj] = v[5];                                                // dc of the children
                pool[e[2] + H + jj] = v[6];
            } else {
#pragma unroll
                for (int k = 0; k < 3; ++k) pool[e[0] + (5 + k) * H + jj] = v[k];          // leaf g_i g_o g_u
            }
        }
        n_dfr = 0;
    };
    // decode (warp 0): up to NB consecutive instructions with the opcode at `at` + their row sources
    auto decode = [&](uint32_t at) {
        flush();
        __syncthreads();
        if (warp == 0) {
            const uint32_t pre_ = chunk[at - cbase], op_ = pre_ & 0xFF;
            const bool head_ = (op_ == HEAD_F || op_ == HEAD_B);
            const uint32_t lim = min(s1, cbase + (uint32_t)CHUNK);
            const uint32_t sz = (uint32_t)words(pre_);
            const uint32_t q = at + (uint32_t)lane * sz;
            const bool ok = lane < NB && q + sz <= lim && (chunk[q - cbase] & 0xFF) == op_;
            const unsigned msk = __ballot_sync(FULLMASK, ok);
            const int nbw = (msk == FULLMASK) ? 32 : (__ffs(~msk) - 1);
            if (lane < nbw) ipos[lane] = (int)(q - cbase);
            if (lane == 0) { bst[0] = nbw; bst[1] = (int)(at + nbw * sz); bst[2] = (int)op_; }
            __syncwarp();
            const float* sp0 = nullptr;
            const float* sp1 = nullptr;
            if (lane < nbw) {           // rows: [h_l; h_r] for internal forward, h for the heads
                const uint32_t* I = chunk + ipos[lane];
                if (op_ == INT_F) { sp0 = pool + I[2]; sp1 = pool + I[3]; }
                else if (head_ && holds_head) sp0 = pool + I[2];
            }
            if (lane < NB) { segp[2 * lane] = sp0; segp[2 * lane + 1] = sp1; }
        }
        __syncthreads();
    };
    // cell operands k0 <= k < k1 of every (node, unit) of the decoded batch -> cin (cp.async, 4 B)
    auto stage_cin = [&](uint32_t op_, int nb_, int k0, int k1) {
        const int kk = k1 - k0;
        for (int i = tid; i < nb_ * UM * kk; i += NTH) {
            const int n = i / (UM * kk), rem = i - n * (UM * kk);
            const int uu = rem / kk, k = k0 + rem - uu * kk;
            cp_async4(cin + (n * UM + uu) * CINMAX + k, cin_src<H>(op_, chunk + ipos[n], k, lc + uu * NCL, pool), 4u);
        }
    };
    // before the barrier wait: operands this CTA wrote itself (children's c; c, gates and dc of a node)
    auto stage_pre = [&]() {
        const uint32_t op_ = (uint32_t)bst[2];
        const int nb_ = bst[0];
        if (op_ == INT_F) stage_cin(op_, nb_, 0, 2);
        else if (op_ == INT_B || op_ == LEAF_B) stage_cin(op_, nb_, 1, n_cin(op_));
    };
    // after it: data written by the other CTAs of the cluster (h rows, dh)
    auto stage_post = [&]() {
        const uint32_t op_ = (uint32_t)bst[2];
        const int nb_ = bst[0];
        if (op_ == INT_B || op_ == LEAF_B) { stage_cin(op_, nb_, 0, 1); return; }
        const bool head_ = (op_ == HEAD_F || op_ == HEAD_B);
        if (head_ && !holds_head) return;
        const int KPr = op_ == INT_F ? LB::KP : LA::KP;
        const int q4 = KPr / 4;
        const int A = H, B = op_ == INT_F ? H : 0;
        for (int i = tid; i < nb_ * q4; i += NTH) {
            const int n = i / q4, c = (i - n * q4) * 4;
            const float* src = nullptr;
            if (c < A) { const float* b = segp[2 * n]; if (b) src = b + c; }
            else if (c < A + B) { const float* b = segp[2 * n + 1]; if (b) src = b + (c - A); }
            cp_async16(xs + n * KPr + c, src ? src : pool, src ? 16u : 0u);
        }
    };
    while (pos < s1) {
        if (pos + 640 > cbase + CHUNK && cbase + CHUNK < s1) refill(pos);
        const uint32_t pre = chunk[pos - cbase];
        const uint32_t op = pre & 0xFF;
        if (op == S) {            // signal (L165): arrive on the cluster barrier, release our writes
            mark(6);
            if (prof && tid == 0) {
                prof[2 + 3 * (pre >> 8)] = gtimer();
                uint64_t* o = prof + 2 + 3 * (S_[1] + 1) + 10 + 10 * (pre >> 8);
#pragma unroll
                for (int k = 0; k < 10; ++k) o[k] = sec[k];
            }
            cluster_arrive();
            pending = true;
            ++pos;
            mark(8);
            flush();
            // between arrive and wait (L165: independent work may sit between a signal and its wait):
            // decode the next batch and stage the operands this CTA produced itself
            if (pos < s1 && (chunk[pos - cbase] & 0xFF) == W) {
                const uint32_t wpre = chunk[pos - cbase];
                uint32_t nx = pos + 1;
                if (nx < s1 && nx + 640 > cbase + CHUNK && cbase + CHUNK < s1) refill(nx);
                bool ahead = false;
                if (nx < s1) { const uint32_t nop = chunk[nx - cbase] & 0xFF; ahead = nop != S && nop != W && nop != LEAF_F; }
                if (ahead) { mark(0); decode(nx); mark(1); stage_pre(); }
                mark(7);
                if (prof && tid == 0) prof[3 + 3 * (wpre >> 8)] = gtimer();
                cluster_wait();
                pending = false;
                if (prof && tid == 0) prof[4 + 3 * (wpre >> 8)] = gtimer();
                pos = nx;
                predecoded = ahead;
            }
            continue;
        }
        if (op == W) {            // wait (L165): all 16 CTAs of the replica have signalled
            mark(7);
            if (prof && tid == 0) prof[3 + 3 * (pre >> 8)] = gtimer();
            cluster_wait();
            pending = false;
            if (prof && tid == 0) prof[4 + 3 * (pre >> 8)] = gtimer();
            ++pos;
            continue;
        }
        if (op == LEAF_F) {       // leaf cells were computed by vpps_leaf_fwd (one GEMM over all leaves)
            pos += 3;
            continue;
        }
        const bool is_head = (op == HEAD_F || op == HEAD_B);
        const bool fwd = (op & 1) == 0;
        const bool kindB = (op == INT_F || op == INT_B);
        const int KP = kindB ? LB::KP : LA::KP;
        if (!predecoded) { mark(0); decode(pos); mark(1); stage_pre(); }
        predecoded = false;
        const int nb = bst[0];
        const uint32_t p = (uint32_t)bst[1];
        mark(1);
        stage_post();
        cp_async_wait_all();
        __syncthreads();

        mark(is_head ? 5 : (fwd ? 2 : 3));
        if (is_head) {            // loss heads (L42) on the CTA holding W_out
            if (holds_head) {
                if (op == HEAD_F) {
                    for (int pi = warp; pi < nb * C; pi += NTH / 32) {
                        const int n = pi / C, c = pi - n * C;
                        float s = 0.f;
                        for (int k = 4 * lane; k < H; k += 128) {
                            const float4 w4 = *reinterpret_cast<const float4*>(Wo + c * H + k);
                            const float4 h4 = *reinterpret_cast<const float4*>(xs + n * KP + k);
                            s += w4.x * h4.x + w4.y * h4.y + w4.z * h4.z + w4.w * h4.w;
                        }
                        s = warp_sum(s);
                        if (lane == 0) zs[n * ZC + c] = s + bo[c];
                    }
                    __syncthreads();
                    for (int n = warp; n < nb; n += NTH / 32) {
                        const uint32_t* I = chunk + ipos[n];
                        const float zl = lane < C ? zs[n * ZC + lane] : -INFINITY;
                        const float m = warp_max(zl);
                        const float lse = m + logf(warp_sum(lane < C ? expf(zl - m) : 0.f));
                        if (lane < C) pool[I[1] + lane] = expf(zl - lse);
                        const float zy = __shfl_sync(FULLMASK, zl, (int)I[3]);
                        if (lane == 0) {
                            pool[I[1] + C] = lse - zy;
                            atomicAdd(pool + P.loss_word, lse - zy);   // aggregated loss node (L205)
                        }
                    }
                } else {
                    for (int i = tid; i < nb * C; i += NTH) {
                        const int n = i / C, c = i - n * C;
                        const uint32_t* I = chunk + ipos[n];
                        zs[n * ZC + c] = __ldcg(pool + I[1] + c) - (c == (int)I[4] ? 1.f : 0.f);
                    }
                    __syncthreads();
                    for (int c = tid; c < C; c += NTH) {
                        float s = 0.f;
                        for (int n = 0; n < nb; ++n) s += zs[n * ZC + c];
                        dbo[c] += s;
                    }
                    for (int i = tid; i < C * H; i += NTH) {
                        const int c = i / H, k = i - c * H;
                        float s = 0.f;
                        for (int n = 0; n < nb; ++n) s = fmaf(zs[n * ZC + c], xs[n * KP + k], s);
                        dWo[i] += s;
                    }
                    for (int i = tid; i < nb * (H / 4); i += NTH) {
                        const int n = i / (H / 4), k = (i - n * (H / 4)) * 4;
                        float v4[4] = {0.f, 0.f, 0.f, 0.f};
                        for (int c = 0; c < C; ++c) {
                            const float dzc = zs[n * ZC + c];
                            const float4 w4 = *reinterpret_cast<const float4*>(Wo + c * H + k);
                            v4[0] = fmaf(w4.x, dzc, v4[0]); v4[1] = fmaf(w4.y, dzc, v4[1]);
                            v4[2] = fmaf(w4.z, dzc, v4[2]); v4[3] = fmaf(w4.w, dzc, v4[3]);
                        }
                        red_add<4>(pool + chunk[ipos[n] + 3] + k, v4);
                    }
                }
            }
            pos = p;
            continue;
        }

        if (fwd) {
            // ---- forward of internal cells: matvec from registers (L123), 4 nodes at a time; the unit's
            //      16 lanes reduce with a transposed butterfly and the lane holding node n's gates does its
            //      cell update ----
            for (int n0 = 0; n0 < nb; n0 += 4) {
                float2 a[4][5];
#pragma unroll
                for (int n = 0; n < 4; ++n)
#pragma unroll
                    for (int o = 0; o < 5; ++o) a[n][o] = make_float2(0.f, 0.f);
#pragma unroll
                for (int t = 0; t < LB::NT; ++t) {
                    const int col0 = LB::CG * (tu + TU * t);
                    const int of = col0 < H ? 3 : 4;
#pragma unroll
                    for (int n = 0; n < 4; ++n) {
                        float xv[LB::CG];
                        lds<LB::CG>(xs + (n0 + n) * LB::KP + col0, xv);
#pragma unroll
                        for (int q = 0; q < LB::CG; q += 2) {
                            const float2 x2 = make_float2(xv[q], xv[q + 1]);
                            const int k = t * LB::CG + q;
#pragma unroll
                            for (int r = 0; r < 3; ++r)
                                a[n][r] = __ffma2_rn(make_float2(wb[r][k], wb[r][k + 1]), x2, a[n][r]);
                            const float2 f2 = __ffma2_rn(make_float2(wb[3][k], wb[3][k + 1]), x2, make_float2(0.f, 0.f));
                            if (of == 3) { a[n][3].x += f2.x; a[n][3].y += f2.y; }
                            else { a[n][4].x += f2.x; a[n][4].y += f2.y; }
                        }
                    }
                }
                float g5[5];
#pragma unroll
                for (int o = 0; o < 5; ++o)
                    g5[o] = treduce4_16(a[0][o].x + a[0][o].y, a[1][o].x + a[1][o].y, a[2][o].x + a[2][o].y,
                                        a[3][o].x + a[3][o].y, gl);
                const int n = n0 + (gl >> 2);
                if ((gl & 3) == 0 && n < nb) {
                    const uint32_t rec = chunk[ipos[n] + 1];
                    const float* b = bias + u * 4;
                    const float* cv = cin + (n * UM + u) * CINMAX;
                    const float i = sigm(g5[0] + b[0]), o = sigm(g5[1] + b[1]), uv = tanhf(g5[2] + b[2]);
                    const float fl = sigm(g5[3] + b[3]), fr = sigm(g5[4] + b[3]);
                    const float c = i * uv + fl * cv[0] + fr * cv[1];
                    pool[rec + j] = o * tanhf(c);                  // h: read by every CTA of the cluster
                    uint32_t* e = dfw + (n * UM + u) * DFW;        // the rest only by this CTA / the GEMMs
                    float* v = reinterpret_cast<float*>(e + 3);
                    e[0] = rec;
                    v[0] = c; v[1] = i; v[2] = o; v[3] = uv; v[4] = fl; v[5] = fr;
                }
            }
            n_dfr = nb * UM;
            dfr_op = op;
        } else {
            // ---- backward: cell backward by thread (unit u, node gl); its gate gradients are recorded
            //      in the node's record for the dW GEMM (L185) and broadcast to the unit's lanes ----
            float g[5] = {0.f, 0.f, 0.f, 0.f, 0.f};
            if (gl < nb) {
                const uint32_t* I = chunk + ipos[gl];
                const uint32_t rec = I[1];
                const float* cv = cin + (gl * UM + u) * CINMAX;
                const float dh = cv[0], dc = cv[1], c = cv[2], i = cv[3], o = cv[4], uv = cv[5];
                const float th = tanhf(c);
                const float chat = dc + dh * o * (1.f - th * th);
                g[0] = chat * uv * i * (1.f - i);
                g[1] = dh * th * o * (1.f - o);
                g[2] = chat * i * (1.f - uv * uv);
                uint32_t* e = dfw + (gl * UM + u) * DFW;      // deferred: only this CTA / the GEMMs read these
                float* v = reinterpret_cast<float*>(e + 3);
                e[0] = rec;
                v[0] = g[0]; v[1] = g[1]; v[2] = g[2];
                if (kindB) {
                    const float fl = cv[6], fr = cv[7], cl = cv[8], cr = cv[9];
                    g[3] = chat * cl * fl * (1.f - fl);
                    g[4] = chat * cr * fr * (1.f - fr);
                    e[1] = I[4]; e[2] = I[6];                   // dc of the children (unique parent)
                    v[3] = g[3]; v[4] = g[4]; v[5] = chat * fl; v[6] = chat * fr;
                }
                dbacc[0] += g[0]; dbacc[1] += g[1]; dbacc[2] += g[2]; dbacc[3] += g[3] + g[4];
            }
            n_dfr = nb * UM;
            dfr_op = op;
            mark(4);
            // transposed products of internal nodes (L94, fn4): per node, dx = Σ_r W[r] g_r over this
            // thread's columns for its unit; the 16 units' slices are summed in shared memory and one
            // vector red.global.add per 4 columns goes into the children's dh.  (Leaves: dX is formed by
            // vpps_leaf_dx after the kernel.)
            if (kindB) {
                const int src = lane & 16;
                for (int n0 = 0; n0 < nb; n0 += NC) {
#pragma unroll
                    for (int dn = 0; dn < NC; ++dn) {
                        const int n = n0 + dn;
                        float gr[5];
#pragma unroll
                        for (int r = 0; r < 5; ++r) gr[r] = __shfl_sync(FULLMASK, g[r], src | (n & 15));
                        float* drow = dxb + (u * NC + dn) * LB::KP;
#pragma unroll
                        for (int t = 0; t < LB::NT; ++t) {
                            const int col0 = LB::CG * (tu + TU * t);
                            const float gf = col0 < H ? gr[3] : gr[4];
                            float dx[LB::CG];
#pragma unroll
                            for (int q = 0; q < LB::CG; q += 2) {
                                const int k = t * LB::CG + q;
                                float2 d = __ffma2_rn(make_float2(wb[0][k], wb[0][k + 1]), make_float2(gr[0], gr[0]),
                                                      make_float2(0.f, 0.f));
                                d = __ffma2_rn(make_float2(wb[1][k], wb[1][k + 1]), make_float2(gr[1], gr[1]), d);
                                d = __ffma2_rn(make_float2(wb[2][k], wb[2][k + 1]), make_float2(gr[2], gr[2]), d);
                                d = __ffma2_rn(make_float2(wb[3][k], wb[3][k + 1]), make_float2(gf, gf), d);
                                dx[q] = d.x;
                                dx[q + 1] = d.y;
                            }
                            sts_granule<LB::CG>(drow + col0, dx, n < nb);
                        }
                    }
                    __syncthreads();
                    constexpr int q4 = LB::KP / 4;
                    for (int i = tid; i < NC * q4; i += NTH) {
                        const int dn = i / q4, c = (i - dn * q4) * 4, n = n0 + dn;
                        if (n >= nb || c >= 2 * H) continue;
                        const uint32_t* I = chunk + ipos[n];
                        float s[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
                        for (int uu = 0; uu < UM; ++uu) {
                            const float4 x = *reinterpret_cast<const float4*>(dxb + (uu * NC + dn) * LB::KP + c);
                            s[0] += x.x; s[1] += x.y; s[2] += x.z; s[3] += x.w;
                        }
                        red_add<4>(c < H ? pool + I[4] + c : pool + I[6] + (c - H), s);
                    }
                    __syncthreads();
                }
            }
        }
        pos = p;
    }
    flush();
    if (pending) cluster_wait();
    mark(8);
    if (prof && tid == 0) {
        prof[1] = gtimer();
        uint64_t* o = prof + 2 + 3 * (S_[1] + 1);
#pragma unroll
        for (int k = 0; k < 10; ++k) o[k] = sec[k];
    }

    // ---- epilogue: bias and head gradients of this replica summed into grads (zeroed by the host);
    //      the weight-matrix gradients come from vpps_dw_gemm (L185) ----
#pragma unroll
    for (int k = 0; k < 4; ++k)
#pragma unroll
        for (int s = 8; s >= 1; s >>= 1) dbacc[k] += __shfl_xor_sync(FULLMASK, dbacc[k], s);
    if (gl == 0) {
#pragma unroll
        for (int k = 0; k < 3; ++k) atomicAdd(P.grads + off[5] + k * H + j, dbacc[k]);
        atomicAdd(P.grads + off[6] + j, dbacc[3]);
    }
    if (holds_head) {
        __syncthreads();
        for (int i = tid; i < C * H; i += NTH) atomicAdd(P.grads + off[4] + i, dWo[i]);
        for (int i = tid; i < C; i += NTH) atomicAdd(P.grads + off[7] + i, dbo[i]);
    }
    // this CTA's records and gradient contributions are complete: count it for the gradient GEMM tiles
    // of its group (release: every thread fences its own writes, then one increment per CTA)
    if (P.done) {
        __threadfence();
        __syncthreads();
        if (tid == 0) atomicAdd(P.done + grp, 1);
    }
}

// ---- dW = Σ_nodes g xᵀ per weight matrix ("concatenate all the left hand side and all the
//      right hand side tensors that participate in the outer-product for each weight matrix, and use
//      dense matrix-matrix multiplication").  Split-K: one CTA per (128 x 64 tile, chunk of KCH nodes);
//      partial tiles are summed into grads (zeroed by the host) with vector L2 reductions; the SGD update
//      (L129, L197) follows as one elementwise pass over the flat parameters ----
struct GemmParams {
    const float* pool;
    const float* inputs;
    float* grads;
    const uint32_t* int_nodes;   // n_int x (rec, rec_l, rec_r), grouped by replica group
    const uint32_t* leaf_nodes;  // n_leaf x (rec, token), grouped by replica group
    int32_t H, E;
    int64_t off[8];
    const float* w_iou;          // W_iou (params), for the leaf input gradient
    float* d_inputs;             // dX, or nullptr
    const int32_t* done;         // per-group completion counters written by vpps_cl / vpps_df (nullptr: no wait)
    int32_t* claim;              // per-group work-claim counters (zeroed per pass), used with `done`
    int32_t done_target;         // CTAs per group
    int32_t n_grp;
    int32_t grp[16];             // groups in processing order (groups expected to finish first go first)
    int32_t int_off[17], leaf_off[17];
    int32_t items[16];           // work items of group g (indexed by group)
    int32_t static_items;        // 1: one CTA per item (waiting on its group) instead of persistent claiming
    uint64_t* trace;             // measurement only: per claimed item (group, item, start ns, end ns, smid)
    // fused tail (persistent mode): once every item is finished (counter fin == total_items) the CTAs
    // apply SGD to the flat parameters in claimed chunks (mode 1) and one CTA copies the summed loss to
    // mapped host memory (loss_dst, may be null)
    int32_t* fin;
    int32_t* tail_claim;
    int32_t total_items;
    int32_t mode;
    float* params;
    int64_t n_floats;
    float lr, wd;
    const float* loss_src;
    float* loss_dst;
    int32_t tc;                  // 1: weight-gradient tiles on the tensor cores (tcgen05, 3xTF32, TMEM)
};

constexpr int TM = 128;          // tile rows (gate-gradient rows)
constexpr int TN = 64;           // tile cols (input columns)

#ifndef VPPS_DW_KCH
#define VPPS_DW_KCH 96           // nodes per work item
#endif
#ifndef VPPS_DW_CPS
#define VPPS_DW_CPS 3            // gradient-GEMM CTAs per SM
#endif
constexpr int KCH = VPPS_DW_KCH;          // nodes per work item (split-K)

// work items of one group: job m = 0 dU_iou, 1 dU_fl, 2 dU_fr, 3 dW_iou (split-K over the group's nodes),
// 4 leaf dX (split-K over the 3H gate rows)

// leaf input gradient dX[tok_l] += Σ_r g_l[r] W_iou[r][:] (word vectors are inputs of the
// leaves).  Tile 64 leaves x 64 columns, split-K over the 3H gate rows in chunks of DXK, 4 x 4 per thread.
// The item stages all of its operands with one batch of cp.async (one L2 round trip): the leaf gate
// gradients row-major ([leaf][k], stride DXS ≡ 4 mod 32: conflict-free column reads) and DXK rows of W_iou.
#ifndef VPPS_DW_DXK
#define VPPS_DW_DXK 128          // gate rows per leaf-dX work item
#endif
constexpr int DXM = 64, DXN = 64, DXK = VPPS_DW_DXK, DXS = DXK + 4;
constexpr size_t DW_SMEM = 4 * (size_t)((KCH * TM + KCH * TN) > (DXM * DXS + DXK * DXN) ? (KCH * TM + KCH * TN)
                                                                                          : (DXM * DXS + DXK * DXN));
__device__ __forceinline__ void leaf_dx_tile(const GemmParams& P, const uint32_t* leaf_nodes, int n_leaf, int b,
                                             float* sm, uint32_t* idx) {
    const int tid = threadIdx.x, H = P.H, E = P.E;
    const int tiles_c = E / DXN, tiles_r = (n_leaf + DXM - 1) / DXM;
    const int kc = b / (tiles_r * tiles_c), t = b - kc * (tiles_r * tiles_c);
    const int r0 = (t / tiles_c) * DXM, c0 = (t % tiles_c) * DXN;
    const int k0 = kc * DXK, nk = min(3 * H, k0 + DXK) - k0;
    float* As = sm;                      // [DXM][DXS]
    float* Bs = sm + DXM * DXS;          // [DXK][DXN]
    if (tid < DXM) {
        const int row = r0 + tid;
        idx[2 * tid] = row < n_leaf ? __ldcg(leaf_nodes + 2 * row) : 0xFFFFFFFFu;
        idx[2 * tid + 1] = row < n_leaf ? __ldcg(leaf_nodes + 2 * row + 1) : 0u;
    }
    __syncthreads();
    for (int e = tid; e < DXM * (DXK / 4); e += 256) {
        const int l = e / (DXK / 4), p = (e % (DXK / 4)) * 4;
        const uint32_t rec = idx[2 * l];
        const bool ok = rec != 0xFFFFFFFFu && p < nk;
        cp_async16(As + l * DXS + p, ok ? P.pool + rec + 5 * H + k0 + p : P.pool, ok ? 16u : 0u);
    }
    for (int e = tid; e < nk * (DXN / 4); e += 256) {
        const int k = e / (DXN / 4), p = (e % (DXN / 4)) * 4;
        cp_async16(Bs + k * DXN + p, P.w_iou + (int64_t)(k0 + k) * E + c0 + p, 16u);
    }
    cp_async_wait_all();
    __syncthreads();
    const int ty = tid / 16, tx = tid % 16;          // leaves r0 + ty + 16a, columns c0 + 4tx .. +3
    float2 acc2[4][2];
#pragma unroll
    for (int a = 0; a < 4; ++a) acc2[a][0] = acc2[a][1] = make_float2(0.f, 0.f);
    // 4 k per step: one LDS.128 per leaf (its 4 gate gradients) and one per k of W_iou (4 columns)
    // (nk is a multiple of 4: chunks of DXK = 128 of the 3H gate rows)
#pragma unroll 2
    for (int k = 0; k < nk; k += 4) {
        float4 av[4];
#pragma unroll
        for (int a = 0; a < 4; ++a) av[a] = *reinterpret_cast<const float4*>(As + (ty + 16 * a) * DXS + k);
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const float4 bv = *reinterpret_cast<const float4*>(Bs + (k + q) * DXN + tx * 4);
            const float2 b01 = make_float2(bv.x, bv.y), b23 = make_float2(bv.z, bv.w);
#pragma unroll
            for (int a = 0; a < 4; ++a) {
                const float g = q == 0 ? av[a].x : q == 1 ? av[a].y : q == 2 ? av[a].z : av[a].w;
                const float2 aa = make_float2(g, g);
                acc2[a][0] = __ffma2_rn(aa, b01, acc2[a][0]);
                acc2[a][1] = __ffma2_rn(aa, b23, acc2[a][1]);
            }
        }
    }
#pragma unroll
    for (int a = 0; a < 4; ++a) {
        const int l = ty + 16 * a;
        const float v[4] = {acc2[a][0].x, acc2[a][0].y, acc2[a][1].x, acc2[a][1].y};
        if (r0 + l < n_leaf) red_add<4>(P.d_inputs + (int64_t)idx[2 * l + 1] * E + c0 + tx * 4, v);
    }
}

constexpr int KTC = 48;          // nodes per tensor-core work item (6 MMA k-steps of 8)

__host__ __device__ inline int job_items(int m, int n_int, int n_leaf, int H, int E, bool dx, bool tc = false) {
    const int kch = tc ? KTC : KCH;
    const int ki = (n_int + kch - 1) / kch, kl = (n_leaf + kch - 1) / kch;
    switch (m) {
        case 0: return (3 * H / TM) * (2 * H / TN) * ki;
        case 1:
        case 2: return (H / TM) * (H / TN) * ki;
        case 3: return (3 * H / TM) * (E / TN) * kl;
        default: return (dx && n_leaf > 0) ? ((n_leaf + DXM - 1) / DXM) * (E / DXN) * ((3 * H + DXK - 1) / DXK) : 0;
    }
}

// ---- tensor-core weight-gradient tile (tcgen05.mma kind::tf32, accumulator in TMEM) ----
// D[128 gate rows][64 input cols] = Σ_k g_k[rows] x_k[cols]ᵀ over <= KTC nodes.  FP32 accuracy with 3xTF32:
// D = A·B + A·B_lo + A_lo·B, where the tensor core truncates A, B to TF32 and A_lo = A - trunc(A) (exact in
// FP32); the dropped A_lo·B_lo term is ~2^-20 of |A||B| (tools/umma_test.cu: 7e-7 max relative error).
// Operands are staged K-major in the SWIZZLE_NONE canonical layout: core matrix = 8 rows x 16 B (4 k),
// rows 16 B apart, SBO = 128 B between 8-row groups, LBO = (rows / 8) * 128 B between 4-k chunks
// (tools/umma_test.cu pins this layout; the MN-major form read zeros on sm_100a).
__shared__ uint32_t tc_tmem;                  // TMEM base of this CTA's 64-column accumulator
__shared__ __align__(8) uint64_t tc_mbar;      // MMA-completion mbarrier
__shared__ uint32_t tc_phase;                 // parity of the next completion

__device__ __forceinline__ uint64_t umma_desc(uint32_t saddr, uint32_t lbo) {
    return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
           ((uint64_t)(128 >> 4) << 32) | ((uint64_t)1 << 46);
}
constexpr uint32_t umma_idesc(int m, int n) {      // F32 accumulate, TF32 A/B, both K-major
    return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(m >> 4) << 24);
}
__device__ __forceinline__ void umma_tf32(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, int acc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
                 "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}\n"
                 ::"r"(d), "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ float tf32_lo(float v) { return v - __uint_as_float(__float_as_uint(v) & 0xFFFFE000u); }

__device__ void tc_setup() {                   // warp 0: TMEM allocation; thread 0: mbarrier
    if (threadIdx.x < 32) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&tc_tmem)), "r"(64));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&tc_mbar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
        tc_phase = 0;
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ void tc_teardown() {
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tc_tmem), "r"(64));
}

__device__ __forceinline__ void dw_item_tc(const GemmParams& P, int m, int b, int n_int, int n_leaf,
                                           const uint32_t* int_nodes, const uint32_t* leaf_nodes, float* sm,
                                           uint32_t* idx) {
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, H = P.H, E = P.E;
    const int rows = (m == 0 || m == 3) ? 3 * H : H;
    const int cols = m == 0 ? 2 * H : (m == 3 ? E : H);
    const int K = m == 3 ? n_leaf : n_int;
    const int tiles_r = rows / TM, tiles_c = cols / TN;
    const int kc = b / (tiles_r * tiles_c), t = b - kc * (tiles_r * tiles_c);
    const int r0 = (t / tiles_c) * TM, c0 = (t % tiles_c) * TN;
    const int k0 = kc * KTC, nk = min(K, k0 + KTC) - k0;
    const int ks = (nk + 7) / 8;                   // MMA k-steps
    const uint32_t ph = tc_phase;                  // read before the staging barrier; thread 0 flips it after
    const int goff = m == 0 ? 7 * H : (m == 1 ? 10 * H : (m == 2 ? 11 * H : 5 * H));
    // smem: A hi/lo [TM x KTC], B hi/lo [TN x KTC], K-major canonical
    float* Ah = sm;
    float* Al = Ah + TM * KTC;
    float* Bh = Al + TM * KTC;
    float* Bl = Bh + TN * KTC;
    constexpr uint32_t LBO_A = (TM / 8) * 128, LBO_B = (TN / 8) * 128;   // bytes between 4-k chunks
    if (tid < nk) {
        const int node = k0 + tid;
        if (m == 3) {
            idx[3 * tid] = __ldcg(leaf_nodes + 2 * node);
            idx[3 * tid + 1] = __ldcg(leaf_nodes + 2 * node + 1);
        } else {
            idx[3 * tid] = __ldcg(int_nodes + 3 * node);
            idx[3 * tid + 1] = __ldcg(int_nodes + 3 * node + 1);
            idx[3 * tid + 2] = __ldcg(int_nodes + 3 * node + 2);
        }
    }
    __syncthreads();
    // A blocks (TM/4 x ks*2), then B blocks (TN/4 x ks*2); k >= nk zero-filled up to the k-step
    const int kb = 2 * ks;                         // 4-k chunks
    const int na = (TM / 4) * kb, nbk = (TN / 4) * kb;
    // every block's loads in flight before any conversion (one L2 round trip): <= 3 blocks per thread
    constexpr int BPT = ((TM / 4) * (2 * KTC / 8) + (TN / 4) * (2 * KTC / 8) + 255) / 256;
    float4 v[BPT][4];
#pragma unroll
    for (int q = 0; q < BPT; ++q) {
        const int e = tid + 256 * q;
        const bool isA = e < na;
        const int ee = isA ? e : e - na;
        const int nr4 = isA ? TM / 4 : TN / 4;      // consecutive threads: consecutive row blocks of one
        const int k4 = ee / nr4, r4 = ee - k4 * nr4; // 4-k chunk (coalesced loads, conflict-free 16 B stores)
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const int k = 4 * k4 + j;
            const float* src = nullptr;
            if (e < na + nbk && k < nk) {
                if (isA) {
                    src = P.pool + idx[3 * k] + goff + r0 + 4 * r4;
                } else {
                    const int c = c0 + 4 * r4;
                    if (m == 3) src = P.inputs + (int64_t)idx[3 * k + 1] * E + c;
                    else if (m == 0) src = c < H ? P.pool + idx[3 * k + 1] + c : P.pool + idx[3 * k + 2] + (c - H);
                    else src = P.pool + idx[3 * k + (m == 1 ? 1 : 2)] + c;
                }
            }
            v[q][j] = src ? __ldcg(reinterpret_cast<const float4*>(src)) : make_float4(0.f, 0.f, 0.f, 0.f);
        }
    }
#pragma unroll
    for (int q = 0; q < BPT; ++q) {
        const int e = tid + 256 * q;
        if (e >= na + nbk) break;
        const bool isA = e < na;
        const int ee = isA ? e : e - na;
        const int nr4 = isA ? TM / 4 : TN / 4;
        const int k4 = ee / nr4, r4 = ee - k4 * nr4;
        float* hi = isA ? Ah : Bh;
        float* lo = isA ? Al : Bl;
        const uint32_t lbo_f = isA ? LBO_A / 4 : LBO_B / 4;
#pragma unroll
        for (int c = 0; c < 4; ++c) {
            const int r = 4 * r4 + c;
            const uint32_t o = (uint32_t)((r >> 3) * 32 + (r & 7) * 4 + k4 * lbo_f);   // floats
            const float a0 = c == 0 ? v[q][0].x : c == 1 ? v[q][0].y : c == 2 ? v[q][0].z : v[q][0].w;
            const float a1 = c == 0 ? v[q][1].x : c == 1 ? v[q][1].y : c == 2 ? v[q][1].z : v[q][1].w;
            const float a2 = c == 0 ? v[q][2].x : c == 1 ? v[q][2].y : c == 2 ? v[q][2].z : v[q][2].w;
            const float a3 = c == 0 ? v[q][3].x : c == 1 ? v[q][3].y : c == 2 ? v[q][3].z : v[q][3].w;
            *reinterpret_cast<float4*>(hi + o) = make_float4(a0, a1, a2, a3);
            *reinterpret_cast<float4*>(lo + o) = make_float4(tf32_lo(a0), tf32_lo(a1), tf32_lo(a2), tf32_lo(a3));
        }
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic smem writes -> tensor core
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    if (tid == 0) {
        constexpr uint32_t idesc = umma_idesc(TM, TN);
        const uint32_t a0 = smem_u32(Ah), al0 = smem_u32(Al), b0 = smem_u32(Bh), bl0 = smem_u32(Bl);
        for (int s = 0; s < ks; ++s) {
            const uint64_t a = umma_desc(a0 + 2 * s * LBO_A, LBO_A), al = umma_desc(al0 + 2 * s * LBO_A, LBO_A);
            const uint64_t bb = umma_desc(b0 + 2 * s * LBO_B, LBO_B), bl = umma_desc(bl0 + 2 * s * LBO_B, LBO_B);
            umma_tf32(tc_tmem, a, bb, idesc, s > 0);
            umma_tf32(tc_tmem, a, bl, idesc, 1);
            umma_tf32(tc_tmem, al, bb, idesc, 1);
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&tc_mbar)) : "memory");
    }
    {
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}\n"
                         : "=r"(ok) : "r"(smem_u32(&tc_mbar)), "r"(ph) : "memory");
    }
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    // epilogue: warp w reads TMEM lanes 32 (w % 4) .. +31 (tile rows), columns 32 (w / 4) .. +31
    const int row = 32 * (warp & 3) + lane, cb = 32 * (warp >> 2);
    uint32_t r[32];
    const uint32_t ta = tc_tmem + ((uint32_t)(32 * (warp & 3)) << 16) + cb;
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
                   "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
                 : "r"(ta));
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                 : "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
                   "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
                 : "r"(ta + 16));
    asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");   // TMEM reads done before the next MMA
    if (tid == 0) tc_phase ^= 1u;
    // transpose through shared memory (the MMA has finished reading the operands) so that a warp's vector
    // reductions cover whole 256-byte row segments: tile [TM][TN + 4]
    constexpr int DS = TN + 4;
    float* Ds = sm;
#pragma unroll
    for (int q = 0; q < 8; ++q)
        *reinterpret_cast<float4*>(Ds + row * DS + cb + 4 * q) =
            make_float4(__uint_as_float(r[4 * q]), __uint_as_float(r[4 * q + 1]), __uint_as_float(r[4 * q + 2]),
                        __uint_as_float(r[4 * q + 3]));
    __syncthreads();
    const int ty = tid / 16, tx = tid % 16;
    float* base = P.grads + P.off[m == 3 ? 0 : m + 1] + (int64_t)r0 * cols + c0 + 4 * tx;
#pragma unroll
    for (int a = 0; a < TM / 16; ++a) {
        const float4 x = *reinterpret_cast<const float4*>(Ds + (ty + 16 * a) * DS + 4 * tx);
        const float v[4] = {x.x, x.y, x.z, x.w};
        red_add<4>(base + (int64_t)(ty + 16 * a) * cols, v);
    }
}

// One work item of group g: item i -> (job m, local index b).  dW tiles: 128 gate rows x 64 input columns
// over the item's <= KCH nodes, all operand rows staged by one batch of cp.async after the node record
// offsets are read once into shared memory; 8 x 4 FFMA2 per thread; partial tile added to grads.
template <bool TC>
__device__ __forceinline__ void dw_item(const GemmParams& P, int g, int i, float* sm, uint32_t* idx) {
    const int tid = threadIdx.x, H = P.H, E = P.E;
    const int n_int = P.int_off[g + 1] - P.int_off[g], n_leaf = P.leaf_off[g + 1] - P.leaf_off[g];
    const uint32_t* int_nodes = P.int_nodes + 3 * P.int_off[g];
    const uint32_t* leaf_nodes = P.leaf_nodes + 2 * P.leaf_off[g];
    int m = 0, b = i;
    while (m < 5) {
        const int n = job_items(m, n_int, n_leaf, H, E, P.d_inputs != nullptr, TC);
        if (b < n) break;
        b -= n;
        ++m;
    }
    if (m == 5) return;
    if (m == 4) { leaf_dx_tile(P, leaf_nodes, n_leaf, b, sm, idx); return; }
    if constexpr (TC) { dw_item_tc(P, m, b, n_int, n_leaf, int_nodes, leaf_nodes, sm, idx); return; }
    const int rows = (m == 0 || m == 3) ? 3 * H : H;
    const int cols = m == 0 ? 2 * H : (m == 3 ? E : H);
    const int K = m == 3 ? n_leaf : n_int;
    const int tiles_r = rows / TM, tiles_c = cols / TN;
    const int kc = b / (tiles_r * tiles_c), t = b - kc * (tiles_r * tiles_c);
    const int r0 = (t / tiles_c) * TM, c0 = (t % tiles_c) * TN;
    const int k0 = kc * KCH, nk = min(K, k0 + KCH) - k0;
    const int goff = m == 0 ? 7 * H : (m == 1 ? 10 * H : (m == 2 ? 11 * H : 5 * H));
    float* Gs = sm;                      // [KCH][TM]
    float* Xs = sm + KCH * TM;           // [KCH][TN]
    // node operands: idx[3k] = g row base, idx[3k+1] / idx[3k+2] = x row bases (left / right or token)
    if (tid < nk) {
        const int node = k0 + tid;
        if (m == 3) {
            idx[3 * tid] = __ldcg(leaf_nodes + 2 * node);
            idx[3 * tid + 1] = __ldcg(leaf_nodes + 2 * node + 1);
        } else {
            idx[3 * tid] = __ldcg(int_nodes + 3 * node);
            idx[3 * tid + 1] = __ldcg(int_nodes + 3 * node + 1);
            idx[3 * tid + 2] = __ldcg(int_nodes + 3 * node + 2);
        }
    }
    __syncthreads();
    for (int e = tid; e < nk * (TM / 4); e += 256) {
        const int k = e / (TM / 4), p = (e % (TM / 4)) * 4;
        cp_async16(Gs + k * TM + p, P.pool + idx[3 * k] + goff + r0 + p, 16u);
    }
    for (int e = tid; e < nk * (TN / 4); e += 256) {
        const int k = e / (TN / 4), p = (e % (TN / 4)) * 4, c = c0 + p;
        const float* src;
        if (m == 3) src = P.inputs + (int64_t)idx[3 * k + 1] * E + c;
        else if (m == 0) src = c < H ? P.pool + idx[3 * k + 1] + c : P.pool + idx[3 * k + 2] + (c - H);
        else src = P.pool + idx[3 * k + (m == 1 ? 1 : 2)] + c;
        cp_async16(Xs + k * TN + p, src, 16u);
    }
    cp_async_wait_all();
    __syncthreads();
    const int ty = tid / 16, tx = tid % 16;        // rows ty*8 .. +7, cols tx*4 .. +3
    float2 acc[8][2];
#pragma unroll
    for (int a = 0; a < 8; ++a) acc[a][0] = acc[a][1] = make_float2(0.f, 0.f);
#pragma unroll 4
    for (int k = 0; k < nk; ++k) {
        const float4 g0 = *reinterpret_cast<const float4*>(Gs + k * TM + ty * 8);
        const float4 g1 = *reinterpret_cast<const float4*>(Gs + k * TM + ty * 8 + 4);
        const float4 xv = *reinterpret_cast<const float4*>(Xs + k * TN + tx * 4);
        const float ga[8] = {g0.x, g0.y, g0.z, g0.w, g1.x, g1.y, g1.z, g1.w};
        const float2 x01 = make_float2(xv.x, xv.y), x23 = make_float2(xv.z, xv.w);
#pragma unroll
        for (int a = 0; a < 8; ++a) {
            const float2 gg = make_float2(ga[a], ga[a]);
            acc[a][0] = __ffma2_rn(gg, x01, acc[a][0]);
            acc[a][1] = __ffma2_rn(gg, x23, acc[a][1]);
        }
    }
    float* base = P.grads + P.off[m == 3 ? 0 : m + 1];
#pragma unroll
    for (int a = 0; a < 8; ++a) {
        const float v[4] = {acc[a][0].x, acc[a][0].y, acc[a][1].x, acc[a][1].y};
#ifdef VPPS_EXP_STORE
        *reinterpret_cast<float4*>(base + (int64_t)(r0 + ty * 8 + a) * cols + c0 + tx * 4) = make_float4(v[0], v[1], v[2], v[3]);
#else
        red_add<4>(base + (int64_t)(r0 + ty * 8 + a) * cols + c0 + tx * 4, v);
#endif
    }
}

// Persistent CTAs claim work items only from groups whose CTAs have all counted themselves done (no CTA
// ever sits on an SM waiting for a group that is still running); groups are scanned in the host's order.
// Without counters (P.done == nullptr) item = blockIdx.x over the groups in order.
template <bool TC>
__global__ void __launch_bounds__(256, VPPS_DW_CPS) vpps_dw_gemm(const GemmParams P) {
    extern __shared__ __align__(16) float dsm[];
    __shared__ uint32_t idx[3 * KCH];
    __shared__ int pick[3];
    const int tid = threadIdx.x;
    if constexpr (TC) tc_setup();
    if (!P.done || P.static_items) {
        // one item per CTA in the host's group order; with counters, wait for the item's group first
        int b = blockIdx.x;
        for (int q = 0; q < P.n_grp; ++q) {
            const int g = P.grp[q];
            if (b < P.items[g]) {
                if (P.done) {
                    if (tid == 0) {
                        uint32_t v;
                        while (true) {
                            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(P.done + g) : "memory");
                            if ((int)v >= P.done_target) break;
                            __nanosleep(200);
                        }
                    }
                    __syncthreads();
                }
                dw_item<TC>(P, g, b, dsm, idx);
                if constexpr (TC) tc_teardown();
                return;
            }
            b -= P.items[g];
        }
        if constexpr (TC) tc_teardown();
        return;
    }
    // (claiming the group's next item ahead, while the current one runs, was measured slower: at the
    // end the last group's items pile up on the CTAs that claimed ahead)
    while (true) {
        if (tid < 32) {
            // lane q looks at group grp[q] (all groups in one parallel round trip); the first eligible
            // group in order is claimed, retrying further groups if its items ran out meanwhile (claiming
            // the newest group first was measured neutral: at the last group's completion every CTA is
            // still busy with earlier items)
            const int lane = tid;
            const int g = lane < P.n_grp ? P.grp[lane] : -1;
            uint32_t c = 0, d = 0;
            if (g >= 0) {
                asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(c) : "l"(P.claim + g) : "memory");
                asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(d) : "l"(P.done + g) : "memory");
            }
            const bool left = g >= 0 && (int)c < P.items[g];
            unsigned ready = __ballot_sync(FULLMASK, left && (int)d >= P.done_target);
            int got_g = -1, got_i = -1;
            while (ready && got_g < 0) {
                const int q = __ffs(ready) - 1;
                int i = 0;
                if (lane == q) i = atomicAdd(P.claim + g, 1);
                i = __shfl_sync(FULLMASK, i, q);
                const int gq = __shfl_sync(FULLMASK, g, q);
                if (i < P.items[gq]) { got_g = gq; got_i = i; }
                ready &= ready - 1;
            }
            const unsigned any_left = __ballot_sync(FULLMASK, left);
            if (lane == 0) { pick[0] = got_g; pick[1] = got_i; pick[2] = any_left != 0; }
        }
        __syncthreads();
        const int g = pick[0], i = pick[1], rem = pick[2];
        __syncthreads();
        if (g >= 0) {
            const uint64_t t0 = P.trace ? gtimer() : 0;
            dw_item<TC>(P, g, i, dsm, idx);
            // the item's reductions into grads / dX are ordered before the count by the barrier and
            // thread 0's release (cumulative), as the SGD tail acquires `fin`
            __syncthreads();
            if (tid == 0) asm volatile("red.release.gpu.global.add.s32 [%0], 1;" ::"l"(P.fin) : "memory");
            if (P.trace && tid == 0) {
                int k = 0;
                for (int q = 0; q < g; ++q) k += P.items[q];
                uint64_t* o = P.trace + 5 * (k + i);
                uint32_t smid;
                asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
                o[0] = (uint64_t)g; o[1] = (uint64_t)i; o[2] = t0; o[3] = gtimer(); o[4] = smid;
            }
            continue;
        }
        if (!rem) break;
        __nanosleep(500);
    }
    if constexpr (TC) tc_teardown();
    // ---- fused tail: SGD over the flat parameters (L129, L197) and the loss read-back (L199) ----
    if (tid == 0) {
        uint32_t f;
        while (true) {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(f) : "l"(P.fin) : "memory");
            if ((int)f >= P.total_items) break;
            __nanosleep(200);
        }
    }
    __syncthreads();
    const uint64_t t_tail = P.trace ? gtimer() : 0;
    // chunks of 4 float4 per thread with every load in flight before the first store (a strided
    // load-update-store loop is one L2 round trip per iteration: params may alias grads for the compiler)
    constexpr int CV = 4;                                  // float4 per thread per chunk
    constexpr int64_t CH = 4 * CV * 256;                   // floats per claimed chunk
    const int64_t n_chunks = P.mode == 1 ? (P.n_floats + CH - 1) / CH : 0;
    while (true) {
        if (tid == 0) pick[0] = atomicAdd(P.tail_claim, 1);
        __syncthreads();
        const int64_t c = pick[0];
        __syncthreads();
        if (c == 0 && P.loss_dst && tid == 0) {
            const float l = *reinterpret_cast<const volatile float*>(P.loss_src);
            *reinterpret_cast<volatile float*>(P.loss_dst) = l;
        }
        if (c >= n_chunks) break;
        const int64_t lo = c * CH, n4 = (min(P.n_floats, lo + CH) - lo) / 4;
        float4* p4 = reinterpret_cast<float4*>(P.params + lo);
        const float4* g4 = reinterpret_cast<const float4*>(P.grads + lo);
        const float lr = P.lr, wd = P.wd;
        float4 a[CV], b[CV];
#pragma unroll
        for (int q = 0; q < CV; ++q) {
            const int64_t k = tid + 256 * q;
            if (k < n4) { a[q] = __ldcg(p4 + k); b[q] = __ldcg(g4 + k); }
        }
#pragma unroll
        for (int q = 0; q < CV; ++q) {
            const int64_t k = tid + 256 * q;
            if (k >= n4) break;
            a[q].x -= lr * (b[q].x + wd * a[q].x); a[q].y -= lr * (b[q].y + wd * a[q].y);
            a[q].z -= lr * (b[q].z + wd * a[q].z); a[q].w -= lr * (b[q].w + wd * a[q].w);
            p4[k] = a[q];
        }
    }
    if (P.trace && tid == 0 && blockIdx.x < 1000) {   // tail stamps (measurement): rows 3000 + CTA
        uint32_t smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        uint64_t* o = P.trace + 5 * (3000 + blockIdx.x);
        o[0] = 99; o[1] = blockIdx.x; o[2] = t_tail; o[3] = gtimer(); o[4] = smid;
    }
}

}  // namespace cl
}  // namespace dev

#define VPPS_CLUSTER_VARIANT(H, E) \
    {1, H, E, 16, (const void*)&dev::cl::vpps_cl<H, E>, &dev::cl::CCfg<H, E>::smem_bytes}

static const Variant kClusterVariants[] = {
    VPPS_CLUSTER_VARIANT(256, 256),    // target: binary Tree-LSTM H = E = 256, 16-CTA clusters
};

const Variant* cluster_variants(int32_t* n) {
    *n = (int32_t)(sizeof(kClusterVariants) / sizeof(kClusterVariants[0]));
    return kClusterVariants;
}

void launch_dw_gemm(const float* pool, const float* inputs, float* d_inputs, float* params, float* grads,
                    const uint32_t* int_nodes, const uint32_t* leaf_nodes, int32_t n_grp, const int32_t* int_off,
                    const int32_t* leaf_off, const int32_t* order, int32_t* done, int32_t done_target,
                    bool early, int32_t H, int32_t E, const int64_t* off, int64_t n_floats, int32_t mode, float lr,
                    float wd, cudaStream_t s, uint64_t* trace, const float* loss_src, float* loss_dst) {
    using namespace dev::cl;
    GemmParams g{};
    g.trace = trace;
    g.pool = pool; g.inputs = inputs; g.grads = grads;
    g.int_nodes = int_nodes; g.leaf_nodes = leaf_nodes;
    g.H = H; g.E = E;
    for (int i = 0; i < 8; ++i) g.off[i] = off[i];
    g.w_iou = params + off[0];
    g.d_inputs = d_inputs;
    g.done = done;
    g.claim = done ? done + 16 : nullptr;
    g.fin = done ? done + 32 : nullptr;
    g.tail_claim = done ? done + 33 : nullptr;
    g.mode = mode;
    g.params = params;
    g.n_floats = n_floats;
    g.lr = lr;
    g.wd = wd;
    g.loss_src = loss_src;
    g.loss_dst = loss_dst;
    g.done_target = done_target;
    g.n_grp = n_grp;
    static const int tc_env = getenv("VPPS_DW_TC") ? atoi(getenv("VPPS_DW_TC")) : 0;
    // tensor-core weight-gradient tiles (opt-in: measured 95.5K vs 100.6K samples/s for the FFMA2 tiles,
    // the split-K tiles are bound by operand staging and the cross-group reductions, not by FMA issue)
    g.tc = tc_env && H % TM == 0 && E % TN == 0;
    int items = 0;
    for (int q = 0; q < n_grp; ++q) {
        const int gi = order ? order[q] : q;
        g.grp[q] = gi;
        const int ni = int_off[gi + 1] - int_off[gi], nl = leaf_off[gi + 1] - leaf_off[gi];
        int n = 0;
        for (int m = 0; m < 5; ++m) n += job_items(m, ni, nl, H, E, d_inputs != nullptr, g.tc != 0);
        g.items[gi] = n;
        items += n;
    }
    for (int i = 0; i <= n_grp; ++i) { g.int_off[i] = int_off[i]; g.leaf_off[i] = leaf_off[i]; }
    g.total_items = items;
    static const int stat = getenv("VPPS_DW_STATIC") ? atoi(getenv("VPPS_DW_STATIC")) : 0;   // TEMP A/B
    const bool fused_tail = done && !stat && items > 0 && (n_floats % 4) == 0;
    if (items > 0) {
        cudaLaunchConfig_t cfg = {};
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        attr[0].val.programmaticStreamSerializationAllowed = 1;
        g.static_items = stat;
        cfg.gridDim = dim3(done && !stat ? std::min(items, 148 * VPPS_DW_CPS) : items);   // persistent when claiming
        cfg.blockDim = dim3(256);
        cfg.dynamicSmemBytes = DW_SMEM;
        cfg.stream = s;
        cfg.attrs = attr;
        // Launched after vpps_df has completed.  As a programmatic dependent (its items overlapping the
        // slowest groups, 8 % more samples/s) the dataflow test selection failed intermittently — a wrong
        // loss or weight gradient in about one stress run in 20 (4 of 72), none of 72 without it;
        // until the cause is isolated that launch is opt-in: VPPS_DW_PDL=1 (measurement only).
        static const bool pdl = getenv("VPPS_DW_PDL") && atoi(getenv("VPPS_DW_PDL")) != 0;
        cfg.numAttrs = early && pdl ? 1 : 0;
        if (g.tc) cudaLaunchKernelEx(&cfg, vpps_dw_gemm<true>, g);
        else cudaLaunchKernelEx(&cfg, vpps_dw_gemm<false>, g);
    }
    if (fused_tail) return;                                            // SGD + loss inside the kernel
    if (mode == 1) launch_sgd(params, grads, n_floats, lr, wd, s);   // W -= lr (dW + wd W), every parameter
    if (loss_dst) cudaMemcpyAsync(loss_dst, loss_src, sizeof(float), cudaMemcpyDeviceToDevice, s);
}

// per-device launch attributes of the gradient GEMM (vpps_define_model calls this after cudaSetDevice)
cudaError_t setup_dw_gemm_attrs() {
    using namespace dev::cl;
    cudaError_t e = cudaFuncSetAttribute(vpps_dw_gemm<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)DW_SMEM);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(vpps_dw_gemm<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)DW_SMEM);
    return e;
}

}  // namespace vpps
