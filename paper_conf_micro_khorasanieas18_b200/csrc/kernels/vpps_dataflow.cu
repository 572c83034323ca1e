// VPPS with dataflow synchronisation (sm_100a) — binary Tree-LSTM.
//
// Same work split as the cluster kernel (vpps_cluster.cu): a replica group of 16 CTAs holds every
// recurrent weight matrix once in registers, each CTA owns 16 consecutive hidden
// units, whole graphs are assigned to groups (SPEC S5g) and the leaf level runs as a GEMM before the
// kernel.  What changes is the signal/wait of L165: instead of a barrier per level (whose release has to
// wait for the CTA's outstanding stores, ~1.8K cycles, before the consumer can even start its L2 round
// trip), every value another CTA reads is stored as a single-copy-atomic 64-bit slot {value, epoch} and
// the consumer polls the data itself:
//   HX[node][H]          h of an internal node that has a consumer (parent or loss head)
//   PART[node][m][k][2U] partial transposed products of a parent: CTA k's contribution to the dh of both
//                        children over the U units CTA m owns (m reads its 16 x 2U slots and sums them
//                        in a fixed order — deterministic, no atomics)
//   HD[node][H]          the loss head's contribution to a labelled node's dh
// The epoch is the pass counter, so slots never need clearing.  Without hardware clusters the groups
// are ordinary co-resident CTAs of a cooperative launch: 9 groups on 144 SMs instead of 7 clusters.
#include <type_traits>
#include "vpps_kernel.cuh"
#include "dev_common.cuh"

namespace vpps {
namespace dev {
namespace df {

constexpr int NTH = 256;
constexpr int UMC = 16;        // hidden units per CTA (CTAs per group: NCL = H / 16)
constexpr int CHUNK = 4096;    // program words staged in shared memory
constexpr int NB = 16;         // nodes per batch (LEAF_B: up to NBL)
constexpr int NBL = 64;        // leaves per LEAF_B batch (no shared staging: one (unit, leaf) pair per thread pass)
constexpr int MAXB = 1 + (NB * 9 > NBL * 4 ? NB * 9 : NBL * 4);   // words of the largest batch
constexpr int NC = 2;          // nodes per transposed-product chunk (two chunk buffers; 4 measured slower)
constexpr int ZC = 32;         // classes per head (C <= 32)
constexpr int CINMAX = 10;
constexpr uint32_t NONE = 0xFFFFFFFFu;
// HEAD_FB: the loss head's forward and backward in one batch (L42: softmax-NLL; dz = p - onehot needs
// nothing but the head's own forward), emitted at the labelled cell's forward level
enum : uint32_t { LEAF_B = 0x21, INT_F = 0x22, INT_B = 0x23, HEAD_FB = 0x42 };

__device__ __forceinline__ int entry_words(uint32_t op) {
    switch (op) {
        case INT_F: return 6;    // rec, hx, rec_l, hx_l, rec_r, hx_r
        case INT_B: return 9;    // rec, adj, dsrc, hd, pp, rec_l, adj_l, rec_r, adj_r
        case HEAD_FB: return 5;  // rec, rec_c, label, hx_c, hd_c
        default: return 4;       // LEAF_B: rec, adj, dsrc, hd
    }
}

typedef unsigned long long u64;
__device__ __forceinline__ u64 tagv(float v, uint32_t e) { return ((u64)e << 32) | __float_as_uint(v); }
__device__ __forceinline__ void st_tag(u64* p, float v, uint32_t e) {
    asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" ::"l"(p), "l"(tagv(v, e)) : "memory");
}
// Poll of one slot: a relaxed GPU-scope (morally strong, single-copy atomic) 8-byte load of an aligned slot
// that producers write with one relaxed 8-byte store, so value and epoch arrive together and the race is
// one the PTX memory model defines.  It compiles to the same LDG.E.64.STRONG.GPU as the earlier .cg form
// (profiles/r2_poll_sass.txt) and pipelines like ordinary loads.
__device__ __forceinline__ u64 ld_slot(const u64* p) {
    u64 v;
    asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void ld_slot2(const u64* p, u64& a, u64& b) {
    asm volatile("ld.relaxed.gpu.global.v2.b64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}
// four tagged slots in one 32-byte store (STG.E.ENL2.256.STRONG.GPU; each 8-byte element stays single-copy
// atomic, so every slot's value and tag still arrive together); p is 32-byte aligned
__device__ __forceinline__ void st_tag4(u64* p, const float* v, uint32_t e) {
    asm volatile("st.relaxed.gpu.global.v4.b64 [%0], {%1, %2, %3, %4};"
                 ::"l"(p), "l"(tagv(v[0], e)), "l"(tagv(v[1], e)), "l"(tagv(v[2], e)), "l"(tagv(v[3], e)) : "memory");
}

template <int H, int E>
struct DCfg {
    static constexpr int UM = UMC;                 // hidden units per CTA
    static constexpr int NCL = H / UM;             // CTAs per group (16 at H = 256, 8 at H = 128)
    static constexpr int TU = NTH / UM;            // threads per unit
    static_assert(H % UM == 0 && TU == 16, "dataflow kernel: 16 units per CTA, 16 threads per unit");
    using LB = Lay<2 * H, TU>;                     // internal bundle rows (i, o, u of U_iou; f) over [h_l; h_r]
    static constexpr int KP = LB::KP;              // 2H
    // column granule t of a thread covers h_l iff t < TH, for every thread of the unit (compile-time split)
    static constexpr int TH = H / (LB::CG * TU);
    static_assert(H % (LB::CG * TU) == 0, "h_l / h_r boundary on a granule-round boundary");
    static constexpr int O_X = CHUNK;                               // xs [NB][KP] floats
    static constexpr int O_DXB = O_X + NB * KP;                     // dxb [2][NTH/32][NC][KP] floats / u64 scratch
    static constexpr int DXB = 2 * (NTH / 32) * NC * KP;           // two buffers of 8 warp slices
    static constexpr int O_CIN = O_DXB + DXB;
    static constexpr int O_BIAS = O_CIN + NB * UM * CINMAX;
    static constexpr int O_ZS = O_BIAS + UM * 4;
    // second staging buffers: consecutive batches alternate, so a batch needs no closing barrier
    static constexpr int O_X2 = O_ZS + NB * ZC;
    static constexpr int O_CIN2 = O_X2 + NB * KP;
    static constexpr int O_HEAD = O_CIN2 + NB * UM * CINMAX;
    static_assert(DXB >= 2 * NB * KP && DXB >= 2 * NB * NCL * 2 * UM, "u64 staging fits in dxb");
    static size_t smem_bytes(int32_t C) { return 4 * (size_t)(O_HEAD + 2 * C * H + 2 * C + 8); }
};

// PROF = false (the production instantiation): every trace stamp, section clock and per-batch record folds
// away at compile time (prof is a constant nullptr); PROF = true when vpps_set_profile_buffer is active
template <int H, int E, bool PROF>
__global__ void __launch_bounds__(NTH, 1) vpps_df(const DfParams P) {
    using T = DCfg<H, E>;
    using LB = typename T::LB;
    constexpr int TU = T::TU, UM = T::UM, KP = T::KP, NCL = T::NCL;
    extern __shared__ __align__(16) uint32_t smw[];
    float* sm = reinterpret_cast<float*>(smw);
    uint32_t* chunk = smw;
    float* xs = sm + T::O_X;
    float* dxb = sm + T::O_DXB;
    u64* tbuf = reinterpret_cast<u64*>(sm + T::O_DXB);     // tagged staging (aliases dxb)
    float* cin = sm + T::O_CIN;
    int cbuf = 0;                                          // transposed-product buffer, alternating across batches
    float* bias = sm + T::O_BIAS;
    float* zs = sm + T::O_ZS;
    const int C = P.C;
    float* Wo = sm + T::O_HEAD;
    float* dWo = Wo + C * H;
    float* bo = dWo + C * H;
    float* dbo = bo + C;

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int grp = blockIdx.x / NCL, lc = blockIdx.x % NCL;
    float* pool = P.pool;
    const int64_t* off = P.off;
    uint32_t ep = 0;
    u64* HX = reinterpret_cast<u64*>(pool + P.df_hx);
    u64* PART = reinterpret_cast<u64*>(pool + P.df_part);
    u64* HD = reinterpret_cast<u64*>(pool + P.df_hd);
    const int u = tid / TU, tu = tid % TU, gl = lane & 15;      // unit slot, thread in unit, lane in group
    const int j = lc * UM + u;                                  // hidden unit of this thread (blocked)
    const bool holds_head = (lc == 0);

    if (PROF && P.prof && threadIdx.x == 0) P.prof[(int64_t)blockIdx.x * P.prof_stride + 11] = gtimer();   // entry
    // ---- prologue: this CTA's rows of U_iou, U_fl, U_fr -> registers (L123, L129) ----
    // register slot t of a lane in the upper half-warp holds granule t ^ 1 (lanes l and l ^ 16 hold the same
    // columns of the warp's two units): the transposed product's pair exchange then keeps slot t and sends
    // slot t + 1 in every lane, with no selects (granules t and t ^ 1 sit on the same side of h_l / h_r)
    const int gsw = (lane & 16) ? 1 : 0;
    static_assert(T::TH % 2 == 0, "swapped granule pairs stay on one side of [h_l; h_r]");
    float wb[4][LB::NREG];
#pragma unroll
    for (int r = 0; r < 4; ++r)
#pragma unroll
        for (int t = 0; t < LB::NT; ++t) {
            const int col = LB::CG * (tu + TU * (t ^ gsw));
            const float* src = r < 3 ? P.params + off[1] + (int64_t)(r * H + j) * (2 * H) + col
                                     : (col < H ? P.params + off[2] + (int64_t)j * H + col
                                                : P.params + off[3] + (int64_t)j * H + col - H);
            if constexpr (LB::CG == 4) {
                const float4 v = __ldg(reinterpret_cast<const float4*>(src));
                wb[r][t * 4] = v.x; wb[r][t * 4 + 1] = v.y; wb[r][t * 4 + 2] = v.z; wb[r][t * 4 + 3] = v.w;
            } else {
#pragma unroll
                for (int q = 0; q < LB::CG; ++q) wb[r][t * LB::CG + q] = __ldg(src + q);
            }
        }
    if (tid < UM * 4) {
        const int uu = tid / 4, k = tid % 4, jj = lc * UM + uu;
        bias[tid] = k < 3 ? __ldg(P.params + off[5] + k * H + jj) : __ldg(P.params + off[6] + jj);
    }
    // the loss head runs in every CTA of the group (each needs dz for its own units' dh): W_out, b_out in
    // every CTA; dW_out accumulates this CTA's columns only
    for (int i = tid; i < C * H; i += NTH) { Wo[i] = __ldg(P.params + off[4] + i); dWo[i] = 0.f; }
    for (int i = tid; i < C; i += NTH) { bo[i] = __ldg(P.params + off[7] + i); dbo[i] = 0.f; }
    float dbacc[4] = {0.f, 0.f, 0.f, 0.f};   // bias gradients of unit lc * UM + tid % UM (INT_B mapping)
    float dbleaf[3] = {0.f, 0.f, 0.f};       // ... of unit lc * UM + tid % UM (LEAF_B mapping)
    uint64_t* prof = PROF && P.prof ? P.prof + (int64_t)blockIdx.x * P.prof_stride : nullptr;
    // section clocks (trace only): 0 program, 1 staging, 2 tag wait, 3 forward, 4 cell-bwd, 5 transposed,
    // 6 heads, 7 other
    uint64_t sec[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    uint64_t sec_last = 0;
    int sec_cur = 7;
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
                default: sec[7] += d; break;
            }
            sec_cur = k;
            sec_last = now;
        }
    };
    // ---- program of this group: batches [op | nb << 8, nb entries].  The script was copied before the
    //      leaf grid ran, so its first chunk loads while that grid drains (before griddepcontrol.wait) ----
    const uint32_t* S_ = P.script + P.df_off;
    const uint32_t G = S_[0];
    const uint32_t s0 = 2 + G + S_[1 + grp], s1 = 2 + G + S_[2 + grp];
    uint32_t cbase = s0;
    auto refill = [&](uint32_t from) {
        __syncthreads();
        for (int i = tid; i < CHUNK; i += NTH) chunk[i] = from + i < s1 ? __ldg(S_ + from + i) : 0u;
        __syncthreads();
        cbase = from;
    };
    if (s0 < s1) refill(s0);
    // the leaf records and the pass counter (vpps_leaf_fwd, the preceding grid) are visible from here on
    asm volatile("griddepcontrol.wait;" ::: "memory");
    // the gradient GEMM (programmatic dependent of this grid) may launch from here on: it reads the
    // `done` / claim counters the leaf grid cleared, which is complete and visible once every CTA of this
    // grid has passed the wait above
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    ep = *P.epoch;
    __syncthreads();
    if (prof && tid == 0) { prof[0] = gtimer(); sec_last = clock64(); }
    uint32_t pos = s0;
    int nbatch = 0;
    int xdone = 0;            // fine stamps taken (trace only)
    while (pos < s1) {
        if (pos + MAXB > cbase + CHUNK && cbase + CHUNK < s1) refill(pos);
        mark(0);
        const uint32_t hdr = chunk[pos - cbase];
        const uint32_t op = hdr & 0xFF;
        const int nb = (int)(hdr >> 8);
        const int sz = entry_words(op);
        const uint32_t* ent = chunk + (pos - cbase) + 1;
        const uint32_t next = pos + 1 + nb * sz;
        const bool is_head = op == HEAD_FB;
        ++nbatch;
        // staging buffers of this batch: the other pair than the previous batch's (a thread still computing
        // that batch reads only those); batch b+2 reuses them after batch b+1's staging barrier
        xs = sm + ((nbatch & 1) ? T::O_X : T::O_X2);
        cin = sm + ((nbatch & 1) ? T::O_CIN : T::O_CIN2);
        uint64_t* bt = (prof && tid == 0 && nbatch <= 48 && P.prof_stride >= 16 + 5 * 48) ? prof + 16 + 5 * (nbatch - 1) : nullptr;
        if (bt) { bt[0] = clock64(); bt[4] = op; }
        int rounds = 0;
        // fine stamps (trace only, tid 0, first single-node batch of each kind): prof[256 + k]
        uint64_t* xst = (prof && tid == 0 && P.prof_stride >= 288) ? prof + 256 : nullptr;
        const bool stF = xst && op == INT_F && nb == 1 && !(xdone & 1);
        const bool stB = xst && op == INT_B && nb == 1 && !(xdone & 2);
        const bool stL = xst && op == LEAF_B && !(xdone & 4);
        const bool stBB = xst && op == INT_B && nb >= 12 && !(xdone & 8);     // first big backward batch
        xdone |= (stF ? 1 : 0) | (stB ? 2 : 0) | (stL ? 4 : 0) | (stBB ? 8 : 0);
#define XST(f, k) do { if (f) xst[k] = clock64(); } while (0)
        XST(stF, 16);
        XST(stB, 22);
        XST(stBB, 27);
        mark(1);
        if (op == LEAF_B) {
            // leaf backward, thread (leaf tid / U + 16 p, unit tid % U): consecutive threads read consecutive
            // units of the same slot row (coalesced), own operands and the 17 dh slots straight into
            // registers, cell backward, gate gradients to the record for the W_iou / dX GEMM (L185)
            const int uu = tid % UM, jj = lc * UM + uu;
            for (int n = tid / UM; n < nb; n += NTH / UM) {
                const uint32_t* e = ent + n * sz;
                const uint32_t rec = e[0], dsrc = e[2], hd = e[3];
                const float dc = __ldcg(pool + e[1] + H + jj), c = __ldcg(pool + rec + H + jj);
                const float i = __ldcg(pool + rec + 2 * H + jj), o = __ldcg(pool + rec + 3 * H + jj);
                const float uv = __ldcg(pool + rec + 4 * H + jj);
                const u64* psrc = dsrc != NONE ? PART + ((((int64_t)(dsrc >> 1) * NCL + lc) * NCL) * 2 + (dsrc & 1)) * UM + uu : nullptr;
                const u64* hsrc = hd != NONE ? HD + (int64_t)hd * H + jj : nullptr;
                const u64 none = (u64)ep << 32;
                u64 v[NCL + 1];
#pragma unroll
                for (int k = 0; k < NCL; ++k) v[k] = psrc ? ld_slot(psrc + k * 2 * UM) : none;
                v[NCL] = hsrc ? ld_slot(hsrc) : none;
                XST(stL && n == tid / UM, 12);
                while (true) {
                    bool stale = false;
#pragma unroll
                    for (int k = 0; k < NCL; ++k)
                        if ((uint32_t)(v[k] >> 32) != ep) { stale = true; v[k] = ld_slot(psrc + k * 2 * UM); }
                    if ((uint32_t)(v[NCL] >> 32) != ep) { stale = true; v[NCL] = ld_slot(hsrc); }
                    if (!stale) break;
                    ++rounds;
                }
                XST(stL && n == tid / UM, 13);
                float dh = 0.f;
#pragma unroll
                for (int k = 0; k <= NCL; ++k) dh += __uint_as_float((uint32_t)v[k]);
                const float th = ftanh(c);
                const float chat = dc + dh * o * (1.f - th * th);
                const float g0 = chat * uv * i * (1.f - i), g1 = dh * th * o * (1.f - o), g2 = chat * i * (1.f - uv * uv);
                pool[rec + 5 * H + jj] = g0;
                pool[rec + 6 * H + jj] = g1;
                pool[rec + 7 * H + jj] = g2;
                dbleaf[0] += g0; dbleaf[1] += g1; dbleaf[2] += g2;
                XST(stL && n == tid / UM, 14);
            }
            XST(stL, 15);
            if (bt) { bt[1] = bt[2] = clock64(); bt[4] |= (uint64_t)rounds << 8; }
            mark(4);
            __syncthreads();
            if (bt) bt[3] = clock64();
            pos = next;
            continue;
        }
        if (op == INT_F || is_head) {
            // rows [h_l; h_r] (INT_F) or h of the labelled node (heads), one half row (H values) per
            // (node, side).  Internal children: H tagged slots = H/2 16-byte pieces -> u64 scratch; leaf
            // children (leaf GEMM output): H floats = H/4 pieces straight into xs.  Half rows are spread
            // over the block NTH / (H/2) at a time with shift-only index math.
            constexpr int PPR = H / 2;                     // pieces per tagged half row
            constexpr int RPP = NTH / PPR;                 // half rows per pass
            const int A = op == INT_F ? 2 : 1;
            const int rows = nb * A;
            const int pr = tid % PPR, rsub = tid / PPR;
            uint32_t my_tagged = 0;                        // bit p: pass p's half row is tagged
            if (rows <= 4 * RPP) {
                // small batch (<= 4 passes per thread): tagged pieces straight into registers, checked and
                // converted there — one L2 round trip and one barrier
                u64 ta[4], tb[4];
#pragma unroll
                for (int p = 0; p < 4; ++p) {
                    const int r = rsub + p * RPP;
                    if (r >= rows) break;
                    const int n = A == 2 ? r >> 1 : r, half = A == 2 ? r & 1 : 0;
                    const uint32_t* e = ent + n * sz;
                    const uint32_t hx = op == INT_F ? e[3 + 2 * half] : e[3];
                    if (hx == NONE) {
                        if (pr < H / 4) cp_async16(xs + n * KP + half * H + 4 * pr, pool + (op == INT_F ? e[2 + 2 * half] : e[1]) + 4 * pr, 16u);
                    } else {
                        ld_slot2(HX + (int64_t)hx * H + 2 * pr, ta[p], tb[p]);
                        my_tagged |= 1u << p;
                    }
                }
                XST(stF, 17);
                if (op == INT_F && tid < nb * UM) {        // c_l, c_r of this CTA's units (own records)
                    const int n = tid / UM, uu = tid % UM;
                    const uint32_t* e = ent + n * sz;
                    cp_async4(cin + tid * CINMAX, pool + e[2] + H + lc * UM + uu, 4u);
                    cp_async4(cin + tid * CINMAX + 1, pool + e[4] + H + lc * UM + uu, 4u);
                }
                cp_async_wait_all();
                XST(stF, 18);
                XST(stF, 19);
                if (bt) bt[1] = clock64();
                mark(2);
                while (true) {
                    int stale = 0;
#pragma unroll
                    for (int p = 0; p < 4; ++p) {
                        if (!(my_tagged >> p & 1u)) continue;
                        const int r = rsub + p * RPP;
                        const int n = A == 2 ? r >> 1 : r, half = A == 2 ? r & 1 : 0;
                        const int o = n * KP + half * H + 2 * pr;
                        if ((uint32_t)(ta[p] >> 32) == ep && (uint32_t)(tb[p] >> 32) == ep) {
                            *reinterpret_cast<float2*>(xs + o) = make_float2(__uint_as_float((uint32_t)ta[p]), __uint_as_float((uint32_t)tb[p]));
                            my_tagged &= ~(1u << p);
                        } else {
                            const uint32_t* e = ent + n * sz;
                            const uint32_t hx = op == INT_F ? e[3 + 2 * half] : e[3];
                            ld_slot2(HX + (int64_t)hx * H + 2 * pr, ta[p], tb[p]);
                            ++stale;
                        }
                    }
                    XST(stF && rounds == 0, 20);
                    if (__syncthreads_count(stale) == 0) break;
                    ++rounds;
                }
            } else {
            for (int r = rsub, p = 0; r < rows; r += RPP, ++p) {
                const int n = A == 2 ? r >> 1 : r, half = A == 2 ? r & 1 : 0;
                const uint32_t* e = ent + n * sz;
                const uint32_t hx = op == INT_F ? e[3 + 2 * half] : e[3];
                if (hx == NONE) {
                    if (pr < H / 4) cp_async16(xs + n * KP + half * H + 4 * pr, pool + (op == INT_F ? e[2 + 2 * half] : e[1]) + 4 * pr, 16u);
                } else {
                    cp_async16(tbuf + n * KP + half * H + 2 * pr, HX + (int64_t)hx * H + 2 * pr, 16u);
                    my_tagged |= 1u << p;
                }
            }
            if (op == INT_F && tid < nb * UM) {            // c_l, c_r of this CTA's units (own records)
                const int n = tid / UM, uu = tid % UM;
                const uint32_t* e = ent + n * sz;
                cp_async4(cin + tid * CINMAX, pool + e[2] + H + lc * UM + uu, 4u);
                cp_async4(cin + tid * CINMAX + 1, pool + e[4] + H + lc * UM + uu, 4u);
            }
            cp_async_wait_all();
            __syncthreads();
            if (bt) bt[1] = clock64();
            mark(2);
            // check the epochs, convert fresh pieces; re-fetch pieces of producers that were still behind
            while (true) {
                int stale = 0;
                for (int r = rsub, p = 0; r < rows; r += RPP, ++p) {
                    if (!(my_tagged >> p & 1u)) continue;
                    const int n = A == 2 ? r >> 1 : r, half = A == 2 ? r & 1 : 0;
                    const int o = n * KP + half * H + 2 * pr;
                    const u64 a = tbuf[o], b = tbuf[o + 1];
                    if ((uint32_t)(a >> 32) == ep && (uint32_t)(b >> 32) == ep) {
                        *reinterpret_cast<float2*>(xs + o) = make_float2(__uint_as_float((uint32_t)a), __uint_as_float((uint32_t)b));
                        my_tagged &= ~(1u << p);
                    } else {
                        const uint32_t* e = ent + n * sz;
                        const uint32_t hx = op == INT_F ? e[3 + 2 * half] : e[3];
                        cp_async16(tbuf + o, HX + (int64_t)hx * H + 2 * pr, 16u);
                        ++stale;
                    }
                }
                if (__syncthreads_count(stale) == 0) break;
                ++rounds;
                cp_async_wait_all();
            }
            }
        } else {
            // backward, thread (n = tid / U, uu = tid % U): dh = Σ_k PART[parent][lc][k][side][uu] (+ HD), its
            // own 17 slots polled with relaxed GPU-scope loads, its own operands (dc at adj + H; c i o u fl fr;
            // the children's c — all written by this CTA) loaded into registers alongside; then the cell
            // backward right here: gate gradients to the record (left operands of the gradient GEMM, L185),
            // the children's dc to theirs, and to shared memory for the transposed product (one barrier)
            const int n = tid / UM, uu = tid % UM, jj = lc * UM + uu;
            const bool act = n < nb;
            const uint32_t* e = ent + (act ? n : 0) * sz;
            const uint32_t dsrc = act ? e[2] : NONE, hd = act ? e[3] : NONE;
            float rv[9];
            if (act) {
                rv[0] = pool[e[1] + H + jj];
#pragma unroll
                for (int k = 0; k < 6; ++k) rv[1 + k] = pool[e[0] + (k + 1) * H + jj];
                rv[7] = pool[e[5] + H + jj];
                rv[8] = pool[e[7] + H + jj];
            }
            const u64* psrc = dsrc != NONE ? PART + ((((int64_t)(dsrc >> 1) * NCL + lc) * NCL) * 2 + (dsrc & 1)) * UM + uu : nullptr;
            const u64* hsrc = hd != NONE ? HD + (int64_t)hd * H + jj : nullptr;
            u64 v[NCL + 1];
            const u64 none = (u64)ep << 32;                // an absent source reads as a current 0
#pragma unroll
            for (int k = 0; k < NCL; ++k) v[k] = psrc ? ld_slot(psrc + k * 2 * UM) : none;
            v[NCL] = hsrc ? ld_slot(hsrc) : none;
            XST(stB, 23);
            XST(stB, 24);
            if (bt) bt[1] = clock64();
            mark(2);
            while (true) {
                bool stale = false;
#pragma unroll
                for (int k = 0; k < NCL; ++k)
                    if ((uint32_t)(v[k] >> 32) != ep) { stale = true; v[k] = ld_slot(psrc + k * 2 * UM); }
                if ((uint32_t)(v[NCL] >> 32) != ep) { stale = true; v[NCL] = ld_slot(hsrc); }
                if (!stale) break;
                ++rounds;
            }
            XST(stB, 25);
            mark(4);
            if (act) {
                float dh = 0.f;
#pragma unroll
                for (int k = 0; k <= NCL; ++k) dh += __uint_as_float((uint32_t)v[k]);
                const float dc = rv[0], c = rv[1], i = rv[2], o = rv[3], uv = rv[4], fl = rv[5], fr = rv[6];
                const float th = ftanh(c);
                const float chat = dc + dh * o * (1.f - th * th);
                float g[5];
                g[0] = chat * uv * i * (1.f - i);
                g[1] = dh * th * o * (1.f - o);
                g[2] = chat * i * (1.f - uv * uv);
                g[3] = chat * rv[7] * fl * (1.f - fl);
                g[4] = chat * rv[8] * fr * (1.f - fr);
                const uint32_t rec = e[0];
                pool[e[6] + H + jj] = chat * fl;          // dc of the children (unique parent; own units)
                pool[e[8] + H + jj] = chat * fr;
#pragma unroll
                for (int r = 0; r < 5; ++r) {
                    pool[rec + (7 + r) * H + jj] = g[r];
                    cin[(n * 5 + r) * UM + uu] = g[r];    // (cin of this batch holds the gate gradients)
                }
                dbacc[0] += g[0]; dbacc[1] += g[1]; dbacc[2] += g[2]; dbacc[3] += g[3] + g[4];
            }
            XST(stB, 26);
            __syncthreads();
            XST(stBB, 28);
        }
        if (bt) { bt[2] = clock64(); bt[4] |= (uint64_t)rounds << 8; }

        mark(is_head ? 6 : (op == INT_F ? 3 : 4));
        if (is_head) {
            // loss heads (L42) in every CTA of the group, one warp per labelled node: logits z = W_out h + b_out
            // (lane c keeps z_c), softmax-NLL, dz = p - onehot(y); the dh = W_out^T dz of this CTA's own units
            // goes to its HD slots, which only this CTA's backward of the labelled cell reads (no cross-CTA
            // exchange: every CTA forms dz itself from the staged h).  CTA 0 writes p and the loss.
            for (int n = warp; n < nb; n += NTH / 32) {
                const uint32_t* e = ent + n * sz;
                float z = -INFINITY;
                for (int c = 0; c < C; ++c) {
                    float s = 0.f;
#pragma unroll
                    for (int k = 4 * lane; k < H; k += 128) {
                        const float4 w4 = *reinterpret_cast<const float4*>(Wo + c * H + k);
                        const float4 h4 = *reinterpret_cast<const float4*>(xs + n * KP + k);
                        s += w4.x * h4.x + w4.y * h4.y + w4.z * h4.z + w4.w * h4.w;
                    }
                    s = warp_sum(s);
                    if (lane == c) z = s + bo[c];
                }
                const float m = warp_max(z);
                const float lse = m + logf(warp_sum(lane < C ? expf(z - m) : 0.f));
                const float p = expf(z - lse);
                const int y = (int)e[2];
                const float dz = lane < C ? p - (lane == y ? 1.f : 0.f) : 0.f;
                zs[n * ZC + lane] = dz;
                if (holds_head) {
                    if (lane < C) pool[e[0] + lane] = p;
                    const float zy = __shfl_sync(FULLMASK, z, y);
                    if (lane == 0) {
                        pool[e[0] + C] = lse - zy;
                        atomicAdd(pool + P.loss_word, lse - zy);   // aggregated loss node (L205)
                    }
                }
                const int jh = lc * UM + (lane % UM);
                float dh = 0.f;
                for (int c = 0; c < C; ++c) dh = fmaf(Wo[c * H + jh], __shfl_sync(FULLMASK, dz, c), dh);
                const uint32_t hd = e[4];
                if (hd != NONE && lane < UM) st_tag(HD + (int64_t)hd * H + jh, dh, ep);
            }
            __syncthreads();
            for (int i = tid; i < C * UM; i += NTH) {             // dW_out of this CTA's columns
                const int c = i / UM, k = lc * UM + (i - c * UM);
                float s = 0.f;
                for (int n = 0; n < nb; ++n) s = fmaf(zs[n * ZC + c], xs[n * KP + k], s);
                dWo[c * H + k] += s;
            }
            if (holds_head)
                for (int c = tid; c < C; c += NTH) {
                    float s = 0.f;
                    for (int n = 0; n < nb; ++n) s += zs[n * ZC + c];
                    dbo[c] += s;
                }
        } else if (op == INT_F) {
            // ---- forward of internal cells: matvec from registers (L123), 4 nodes at a time; the unit's
            //      16 lanes reduce with a transposed butterfly; the lane holding node n's gates updates it ----
            // groups of NN in {4, 2, 1} nodes: the unit's 16 lanes reduce NN partial sums with a transposed
            // butterfly, after which lane 16/NN * m holds node m's gates
            auto fwd_group = [&](auto nnc, int n0) {
                constexpr int NN = decltype(nnc)::value;
                XST(stF, 0);
                float2 a[NN][5];
#pragma unroll
                for (int n = 0; n < NN; ++n)
#pragma unroll
                    for (int o = 0; o < 5; ++o) a[n][o] = make_float2(0.f, 0.f);
#pragma unroll
                for (int t = 0; t < LB::NT; ++t) {
                    const int col0 = LB::CG * (tu + TU * (t ^ gsw));
                    constexpr int of0 = 3;                  // granules t < T::TH read h_l (U_fl), the rest h_r (U_fr)
#pragma unroll
                    for (int n = 0; n < NN; ++n) {
                        float xv[LB::CG];
                        lds<LB::CG>(xs + (n0 + n) * KP + col0, xv);
#pragma unroll
                        for (int q = 0; q < LB::CG; q += 2) {
                            const float2 x2 = make_float2(xv[q], xv[q + 1]);
                            const int k = t * LB::CG + q;
#pragma unroll
                            for (int r = 0; r < 3; ++r)
                                a[n][r] = __ffma2_rn(make_float2(wb[r][k], wb[r][k + 1]), x2, a[n][r]);
                            a[n][of0 + (t >= T::TH)] = __ffma2_rn(make_float2(wb[3][k], wb[3][k + 1]), x2, a[n][of0 + (t >= T::TH)]);
                        }
                    }
                }
                XST(stF, 1);
                float g5[5];
#pragma unroll
                for (int o = 0; o < 5; ++o) {
                    if constexpr (NN == 4) {
                        g5[o] = treduce4_16(a[0][o].x + a[0][o].y, a[1][o].x + a[1][o].y, a[2][o].x + a[2][o].y,
                                            a[3][o].x + a[3][o].y, gl);
                    } else if constexpr (NN == 2) {
                        const bool b3 = gl & 8;
                        const float v0 = a[0][o].x + a[0][o].y, v1 = a[1][o].x + a[1][o].y;
                        float k = b3 ? v1 : v0;
                        k += __shfl_xor_sync(FULLMASK, b3 ? v0 : v1, 8);
                        k += __shfl_xor_sync(FULLMASK, k, 4);
                        k += __shfl_xor_sync(FULLMASK, k, 2);
                        g5[o] = k + __shfl_xor_sync(FULLMASK, k, 1);
                    } else {
                        float k = a[0][o].x + a[0][o].y;
#pragma unroll
                        for (int d = 8; d >= 1; d >>= 1) k += __shfl_xor_sync(FULLMASK, k, d);
                        g5[o] = k;
                    }
                }
                XST(stF, 2);
                constexpr int SPAN = 16 / NN;
                const int n = n0 + gl / SPAN;
                if (gl % SPAN == 0 && n < nb) {
                    const uint32_t* e = ent + n * sz;
                    const uint32_t rec = e[0];
                    const float* b = bias + u * 4;
                    const float* cv = cin + (n * UM + u) * CINMAX;
                    const float i = fsigm(g5[0] + b[0]), o = fsigm(g5[1] + b[1]), uv = ftanh(g5[2] + b[2]);
                    const float fl = fsigm(g5[3] + b[3]), fr = fsigm(g5[4] + b[3]);
                    const float c = i * uv + fl * cv[0] + fr * cv[1];
                    const float h = o * ftanh(c);
                    if (e[1] != NONE) st_tag(HX + (int64_t)e[1] * H + j, h, ep);   // read by the whole group
                    pool[rec + j] = h;                                              // the rest: this CTA, GEMMs
                    pool[rec + H + j] = c;
                    pool[rec + 2 * H + j] = i;
                    pool[rec + 3 * H + j] = o;
                    pool[rec + 4 * H + j] = uv;
                    pool[rec + 5 * H + j] = fl;
                    pool[rec + 6 * H + j] = fr;
                }
                XST(stF, 3);
            };
            int n0 = 0;
            for (; n0 + 2 < nb; n0 += 4) fwd_group(std::integral_constant<int, 4>{}, n0);
            if (nb - n0 == 2) fwd_group(std::integral_constant<int, 2>{}, n0);
            else if (nb - n0 == 1) fwd_group(std::integral_constant<int, 1>{}, n0);
        } else {
            // ---- backward: the gate gradients of the batch are in shared memory (cin), from the staging ----
            const bool kindB = op == INT_B;
            mark(5);
            XST(stB, 5);
            XST(stB, 6);
            XST(stBB, 29);
            // transposed products (L94, fn4): per node, this CTA's partial dx = Σ_r W[r] g_r over all 2H
            // columns.  The two units of a warp are pre-summed with one shuffle exchange (lane l keeps the
            // even or odd granules of the pair, l ^ 16 the others), the 8 warp slices are summed in shared
            // memory and published as tagged PART slots.  Chunks of NC nodes alternate between two
            // buffers, so one barrier per chunk separates a chunk's stores from its reduction and the
            // reduction of chunk c overlaps the products of chunk c + 1.
            if (kindB) {
                constexpr int NW = NTH / 32;
                const bool hi = lane & 16;
                for (int n0 = 0; n0 < nb; n0 += NC, cbuf ^= 1) {
                    float* buf = dxb + cbuf * (NW * NC * KP);
#pragma unroll
                    for (int dn = 0; dn < NC; ++dn) {
                        const int n = n0 + dn;
                        if (n >= nb) break;
                        float gr[5];
#pragma unroll
                        for (int r = 0; r < 5; ++r) gr[r] = cin[(n * 5 + r) * UM + u];
                        float* drow = buf + (warp * NC + dn) * KP;
#pragma unroll
                        for (int t = 0; t < LB::NT; t += 2) {
                            // granules t, t + 1; lanes < 16 keep granule t, lanes >= 16 granule t + 1 (the
                            // partner lane l ^ 16 holds the same columns of the warp's other unit)
                            float dx[2][LB::CG];
#pragma unroll
                            for (int h = 0; h < 2; ++h) {
                                const float gf = t + h < T::TH ? gr[3] : gr[4];
#pragma unroll
                                for (int q = 0; q < LB::CG; q += 2) {
                                    const int k = (t + h) * LB::CG + q;
                                    float2 d = __ffma2_rn(make_float2(wb[0][k], wb[0][k + 1]), make_float2(gr[0], gr[0]),
                                                          make_float2(0.f, 0.f));
                                    d = __ffma2_rn(make_float2(wb[1][k], wb[1][k + 1]), make_float2(gr[1], gr[1]), d);
                                    d = __ffma2_rn(make_float2(wb[2][k], wb[2][k + 1]), make_float2(gr[2], gr[2]), d);
                                    d = __ffma2_rn(make_float2(wb[3][k], wb[3][k + 1]), make_float2(gf, gf), d);
                                    dx[h][q] = d.x;
                                    dx[h][q + 1] = d.y;
                                }
                            }
                            float kv[LB::CG];
#pragma unroll
                            for (int q = 0; q < LB::CG; ++q) {
                                // slot t is granule t (t + 1 in the upper half-warp): keep it, send slot t + 1
                                kv[q] = dx[0][q] + __shfl_xor_sync(FULLMASK, dx[1][q], 16);
                            }
                            const int col0 = LB::CG * (tu + TU * (t + (hi ? 1 : 0)));
                            sts_granule<LB::CG>(drow + col0, kv, true);
                        }
                    }
                    XST(stB, 7);
                    __syncthreads();
                    XST(stB, 8);
                    constexpr int q4 = KP / 4;
                    for (int i = tid; i < NC * q4; i += NTH) {
                        const int dn = i / q4, c = (i - dn * q4) * 4, n = n0 + dn;
                        if (n >= nb) continue;
                        float s4[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
                        for (int w = 0; w < NW; ++w) {
                            const float4 x = *reinterpret_cast<const float4*>(buf + (w * NC + dn) * KP + c);
                            s4[0] += x.x; s4[1] += x.y; s4[2] += x.z; s4[3] += x.w;
                        }
                        // column c: child side = c / H, unit jj = c % H, owner CTA m = jj / U, slot jj % U
                        const int side = c >= H, jj = c - side * H, m = jj / UM;
                        const uint32_t pp = ent[n * sz + 4];
                        st_tag4(PART + ((((int64_t)pp * NCL + m) * NCL + lc) * 2 + side) * UM + (jj - m * UM), s4, ep);
                    }
                    XST(stB, 9);
                    XST(stB, 10);
                }
                XST(stBB, 30);
            }
        }
        // (no closing barrier: the next batch stages into the other buffers, and every cross-batch reuse
        //  of shared memory is ordered by a staging or refill barrier in between)
        XST(stF, 4);
        XST(stB, 11);
        XST(stBB, 31);
        if (bt) bt[3] = clock64();
        pos = next;
    }
    mark(7);
    if (prof && tid == 0) {
        prof[1] = gtimer();
        prof[2] = (uint64_t)nbatch;
#pragma unroll
        for (int k = 0; k < 8; ++k) prof[3 + k] = sec[k];
    }

    // ---- epilogue: bias and head gradients of this group summed into grads (zeroed by the host); the
    //      weight-matrix gradients come from vpps_dw_gemm (L185) ----
    // (dbacc: unit lc * UM + tid % UM, like dbleaf: lanes l and l ^ 16 share a unit)
#pragma unroll
    for (int k = 0; k < 4; ++k) dbacc[k] += __shfl_xor_sync(FULLMASK, dbacc[k], 16);
    if (lane < 16) {
#pragma unroll
        for (int k = 0; k < 3; ++k) atomicAdd(P.grads + off[5] + k * H + lc * UM + lane, dbacc[k]);
        atomicAdd(P.grads + off[6] + lc * UM + lane, dbacc[3]);
    }
#pragma unroll
    for (int k = 0; k < 3; ++k) dbleaf[k] += __shfl_xor_sync(FULLMASK, dbleaf[k], 16);   // lanes l, l^16: same unit
    if (lane < 16) {
#pragma unroll
        for (int k = 0; k < 3; ++k) atomicAdd(P.grads + off[5] + k * H + lc * UM + lane, dbleaf[k]);
    }
    __syncthreads();
    for (int i = tid; i < C * UM; i += NTH) {
        const int c = i / UM, k = lc * UM + (i - c * UM);
        atomicAdd(P.grads + off[4] + c * H + k, dWo[c * H + k]);
    }
    if (holds_head)
        for (int i = tid; i < C; i += NTH) atomicAdd(P.grads + off[7] + i, dbo[i]);
    // this CTA's records and gradient contributions are complete: count it for the GEMM tiles of its group
    if (P.done) {
        __threadfence();
        __syncthreads();
        if (tid == 0) atomicAdd(P.done + grp, 1);
    }
    if (prof && tid == 0) prof[12] = gtimer();   // exit
}

}  // namespace df
}  // namespace dev

#define VPPS_DF_VARIANT(H, E) \
    {1, H, E, dev::df::DCfg<H, E>::NCL, (const void*)&dev::df::vpps_df<H, E, false>, &dev::df::DCfg<H, E>::smem_bytes}

static const Variant kDfVariants[] = {
    VPPS_DF_VARIANT(256, 256),    // target: binary Tree-LSTM H = E = 256, groups of 16 CTAs
    VPPS_DF_VARIANT(128, 128),    // H = 128: groups of 8 CTAs (16 groups on 128 SMs)
    VPPS_DF_VARIANT(128, 256),
};

// the profiling instantiation of a dataflow variant (same shared memory, in-kernel trace enabled)
const void* df_prof_fn(const void* fn) {
#define VPPS_DF_PROF(H, E) \
    if (fn == (const void*)&dev::df::vpps_df<H, E, false>) return (const void*)&dev::df::vpps_df<H, E, true>;
    VPPS_DF_PROF(256, 256)
    VPPS_DF_PROF(128, 128)
    VPPS_DF_PROF(128, 256)
#undef VPPS_DF_PROF
    return nullptr;
}

const Variant* df_variants(int32_t* n) {
    *n = (int32_t)(sizeof(kDfVariants) / sizeof(kDfVariants[0]));
    return kDfVariants;
}

}  // namespace vpps
