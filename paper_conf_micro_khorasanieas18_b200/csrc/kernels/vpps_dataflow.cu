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
#include <cstdio>
#include <type_traits>
#include "vpps_kernel.cuh"
#include "dev_common.cuh"

namespace vpps {
namespace dev {
namespace df {

constexpr int UMC = 16;        // hidden units per CTA (CTAs per group: NCL = H / 16)
constexpr int CHUNK = 4096;    // program words staged in shared memory
constexpr int NB = 16;         // nodes per batch (LEAF_B: up to NBL)
constexpr int NBL = 64;        // leaves per LEAF_B batch (no shared staging: one (unit, leaf) pair per thread pass)
constexpr int MAXB = 1 + (NB * 9 > NBL * 4 ? NB * 9 : NBL * 4);   // words of the largest batch
constexpr int NC = 2;          // nodes per transposed-product chunk (two chunk buffers; 4 measured slower)
constexpr int ZC = 32;         // classes per head (C <= 32)
constexpr int CINMAX = 10;
#ifndef VPPS_DF_WARP_STAGE
#define VPPS_DF_WARP_STAGE 1 // INT_F batches staged per warp (only the warp's own columns)
#endif
#ifndef VPPS_DF_CHECK
#define VPPS_DF_CHECK 0      // 1: bounds-checked build (every batch entry against its region; traps)
#endif
#ifndef VPPS_DF_NP
#define VPPS_DF_NP 2         // nodes per transposed-product step
#endif
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
// two adjacent tagged slots in one 16-byte store (p 16-byte aligned)
__device__ __forceinline__ void st_tag2(u64* p, float a, float b, uint32_t e) {
    asm volatile("st.relaxed.gpu.global.v2.b64 [%0], {%1, %2};" ::"l"(p), "l"(tagv(a, e)), "l"(tagv(b, e)) : "memory");
}
// four tagged slots in one 32-byte store (STG.E.ENL2.256.STRONG.GPU; each 8-byte element stays single-copy
// atomic, so every slot's value and tag still arrive together); p is 32-byte aligned
__device__ __forceinline__ void st_tag4(u64* p, const float* v, uint32_t e) {
    asm volatile("st.relaxed.gpu.global.v4.b64 [%0], {%1, %2, %3, %4};"
                 ::"l"(p), "l"(tagv(v[0], e)), "l"(tagv(v[1], e)), "l"(tagv(v[2], e)), "l"(tagv(v[3], e)) : "memory");
}

// Loads of record words (children's c, the INT_B operands): L1-cached by default; VPPS_DF_L2REC=1 routes
// them through L2 (measurement build for the intermittent failure of DESIGN §6)
#ifndef VPPS_DF_L2REC
#define VPPS_DF_L2REC 0
#endif
__device__ __forceinline__ void cin_ld2(float* dst, const float* l, const float* r) {
#if VPPS_DF_L2REC
    const float a = __ldcg(l), b = __ldcg(r);
    dst[0] = a;
    dst[1] = b;
#else
    cp_async4(dst, l, 4u);
    cp_async4(dst + 1, r, 4u);
#endif
}
#if VPPS_DF_L2REC
#define RV_LD(p) __ldcg(p)
#else
#define RV_LD(p) (*(p))
#endif

template <int H, int E>
struct DCfg {
    // threads per CTA (512 threads at 128 registers were measured slower: spills, 112 K vs 129 K samples/s)
    static constexpr int NTH = 256;
    static constexpr int NW = NTH / 32;            // warps per CTA
    static constexpr int UM = UMC;                 // hidden units per CTA
    static constexpr int NCL = H / UM;             // CTAs per group (16 at H = 256, 8 at H = 128)
    static constexpr int TU = NTH / UM;            // threads per unit
    static_assert(H % UM == 0, "dataflow kernel: 16 units per CTA");
    using LB = Lay<2 * H, TU>;                     // internal bundle rows (i, o, u of U_iou; f) over [h_l; h_r]
    static constexpr int KP = LB::KP;              // 2H
    // column granule t of a thread covers h_l iff t < TH, for every thread of the unit (compile-time split)
    static constexpr int TH = H / (LB::CG * TU);
    static_assert(H % (LB::CG * TU) == 0, "h_l / h_r boundary on a granule-round boundary");
    static constexpr int O_X = CHUNK;                               // xs [NB][KP] floats
    static constexpr int O_DXB = O_X + NB * KP;                     // u64 staging of tagged rows (NB x KP slots)
    static constexpr int DXB = 2 * NB * KP;
    static constexpr int O_CIN = O_DXB + DXB;
    static constexpr int O_BIAS = O_CIN + NB * UM * CINMAX;
    static constexpr int O_ZS = O_BIAS + UM * 4;
    // second staging buffers: consecutive batches alternate, so a batch needs no closing barrier
    static constexpr int O_X2 = O_ZS + NB * ZC;
    static constexpr int O_CIN2 = O_X2 + NB * KP;
    // forward partial gate sums of the NW warps (column slices), two buffers: [2][NW][4 nodes][UM][4 rows]
    static constexpr int O_FP = O_CIN2 + NB * UM * CINMAX;
    static constexpr int FPB = NW * 4 * UM * 4;
    static constexpr int O_HEAD = O_FP + 2 * FPB;
    static_assert(DXB >= 2 * NB * KP && DXB >= 2 * NB * NCL * 2 * UM, "u64 staging fits in dxb");
    // register layout (unit pairs x column slices): warp w owns columns [w CW, (w + 1) CW) of [h_l; h_r] for
    // all UM units of the CTA; lane = 4 ug + cg holds units 2 ug, 2 ug + 1 (one float2 per (row, column):
    // FFMA2 over the unit pair) and the CPL columns w CW + 16 t + 4 cg + q (granule t, q < 4)
    static constexpr int CW = KP / NW;             // columns per warp
    static constexpr int CPL = CW / 4;             // columns per lane
    static constexpr int NG = CPL / 4;             // 4-column granules per lane
    static_assert(CPL % 8 == 0 && UM == 16 && (NTH == 256 || NTH == 512),
                  "dataflow kernel: NW warps x (8 unit pairs x 4 column groups), >= 8 columns per lane");
    static size_t smem_bytes(int32_t C) { return 4 * (size_t)(O_HEAD + 2 * C * H + 2 * C + 8); }
};

// PROF = false (the production instantiation): every trace stamp, section clock and per-batch record folds
// away at compile time (prof is a constant nullptr); PROF = true when vpps_set_profile_buffer is active
template <int H, int E, bool PROF>
__global__ void __launch_bounds__(DCfg<H, E>::NTH, 1) vpps_df(const DfParams P) {
    using T = DCfg<H, E>;
    constexpr int NTH = T::NTH, NW = T::NW;
    using LB = typename T::LB;
    constexpr int UM = T::UM, KP = T::KP, NCL = T::NCL;
    extern __shared__ __align__(16) uint32_t smw[];
    float* sm = reinterpret_cast<float*>(smw);
    uint32_t* chunk = smw;
    float* xs = sm + T::O_X;
    u64* tbuf = reinterpret_cast<u64*>(sm + T::O_DXB);     // tagged staging (aliases dxb)
    float* cin = sm + T::O_CIN;
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
    const bool holds_head = (lc == 0);

    if (PROF && P.prof && threadIdx.x == 0) P.prof[(int64_t)blockIdx.x * P.prof_stride + 11] = gtimer();   // entry
    // ---- prologue: this CTA's rows of U_iou, U_fl, U_fr -> registers (L123, L129) ----
    // lane (ug, cg) of warp w: units 2 ug, 2 ug + 1 of this CTA as float2 pairs, rows i, o, u of U_iou and the
    // forget row of the warp's side (U_fl over h_l for w < 4, U_fr over h_r otherwise), columns
    // w CW + 16 t + 4 cg + q
    constexpr int CW = T::CW, CPL = T::CPL, NG = T::NG;
    const int cg = lane & 3, ug = lane >> 2;
    const int side = warp >= NW / 2 ? 1 : 0;                    // the warp's columns read h_l (0) or h_r (1)
    float2 wp[4][CPL];
#pragma unroll
    for (int r = 0; r < 4; ++r)
#pragma unroll
        for (int t = 0; t < NG; ++t) {
            const int col = warp * CW + 16 * t + 4 * cg;
            float4 v[2];
#pragma unroll
            for (int m = 0; m < 2; ++m) {
                const int jm = lc * UM + 2 * ug + m;
                const float* src = r < 3 ? P.params + off[1] + (int64_t)(r * H + jm) * (2 * H) + col
                                         : P.params + off[2 + side] + (int64_t)jm * H + col - side * H;
                v[m] = __ldg(reinterpret_cast<const float4*>(src));
            }
            wp[r][4 * t] = make_float2(v[0].x, v[1].x);
            wp[r][4 * t + 1] = make_float2(v[0].y, v[1].y);
            wp[r][4 * t + 2] = make_float2(v[0].z, v[1].z);
            wp[r][4 * t + 3] = make_float2(v[0].w, v[1].w);
        }
    float* fpb = sm + T::O_FP;     // forward partials, two alternating buffers
    int fbuf = 0;
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
#if VPPS_DF_CHECK
        // checked build (tests only; compute-sanitizer is not available on the pool): every field of the
        // batch within its region before anything is staged — a violation traps (the pass fails loudly)
        {
            const bool okh = (op == INT_F || op == INT_B || op == HEAD_FB) ? (nb >= 1 && nb <= NB)
                           : (op == LEAF_B && nb >= 1 && nb <= NBL);
            if (!okh || next > s1 || 1 + nb * sz > MAXB) {
                if (tid == 0) printf("vpps_df check: CTA %d batch %d op %x nb %d\n", blockIdx.x, nbatch, op, nb);
                __trap();
            }
            // record extents: internal record 12 H (h c i o u fl fr + 5 gate gradients), leaf record 8 H,
            // dc slot at adj + H, head record C + 1 (p, loss)
            auto in = [&](uint32_t r, int64_t ext) { return (int64_t)r + ext <= P.pool_words; };
            auto opt_ok = [&](uint32_t v, int64_t n) { return v == NONE || (int64_t)v < n; };
            for (int i = tid; i < nb; i += NTH) {
                const uint32_t* e = ent + i * sz;
                bool ok = true;
                if (op == INT_F) ok = in(e[0], 12 * H) && in(e[2], 2 * H) && in(e[4], 2 * H) && opt_ok(e[1], P.n_hx) &&
                                      opt_ok(e[3], P.n_hx) && opt_ok(e[5], P.n_hx);
                else if (op == INT_B) ok = in(e[0], 12 * H) && in(e[1], 2 * H) && in(e[5], 2 * H) && in(e[6], 2 * H) &&
                                           in(e[7], 2 * H) && in(e[8], 2 * H) &&
                                           (e[2] == NONE || (int64_t)(e[2] >> 1) < P.n_part) &&
                                           opt_ok(e[3], P.n_hd) && (int64_t)e[4] < P.n_part;
                else if (op == HEAD_FB) ok = in(e[0], C + 1) && in(e[1], H) && (int)e[2] < C && opt_ok(e[3], P.n_hx) &&
                                             opt_ok(e[4], P.n_hd);
                else ok = in(e[0], 8 * H) && in(e[1], 2 * H) && (e[2] == NONE || (int64_t)(e[2] >> 1) < P.n_part) &&
                          opt_ok(e[3], P.n_hd);
                if (!ok) {
                    printf("vpps_df check: CTA %d batch %d op %x entry %d out of range\n", blockIdx.x, nbatch, op, i);
                    __trap();
                }
            }
        }
#endif
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
        if (op == INT_F && VPPS_DF_WARP_STAGE) {
            // per-warp staging: warp w computes only with the CW columns [w CW, (w + 1) CW) of [h_l; h_r], so
            // it loads, checks and converts exactly those (child side = w / (NW / 2)) for every node of the batch into
            // its own slice of xs, with a warp-level retry loop — no CTA barrier before the products (the
            // forward group's barrier orders the children's c below for the cell threads)
            // 16-byte L2-only copies (cp.async.cg; an L1-cached poll could keep returning a stale line): lane l
            // carries tagged piece l (slots 2l, 2l + 1 of the slice) and leaf piece l (floats 4l .. 4l + 3)
            const bool tl = 2 * lane < CW, ll = 4 * lane < CW;
            u64* tw = tbuf + warp * (NB * CW);             // this warp's tagged staging
            const int cs = (warp % (NW / 2)) * CW;         // the slice's first column in the child's h
            uint32_t pend = 0;                             // bit n: node n's slots are tagged and not yet converted
            for (int n = 0; n < nb; ++n) {
                const uint32_t* e = ent + n * sz;
                const uint32_t hx = e[3 + 2 * side];
                if (hx == NONE) {
                    if (ll) cp_async16(xs + n * KP + warp * CW + 4 * lane, pool + e[2 + 2 * side] + cs + 4 * lane, 16u);
                } else {
                    if (tl) cp_async16(tw + n * CW + 2 * lane, HX + (int64_t)hx * H + cs + 2 * lane, 16u);
                    pend |= 1u << n;
                }
            }
            if (!tl) pend = 0;
            XST(stF, 17);
            if (tid < nb * UM) {                           // c_l, c_r of this CTA's units (own records)
                const int n = tid / UM, uu = tid % UM;
                const uint32_t* e = ent + n * sz;
                cin_ld2(cin + tid * CINMAX, pool + e[2] + H + lc * UM + uu, pool + e[4] + H + lc * UM + uu);
            }
            cp_async_wait_all();
            XST(stF, 18);
            if (bt) bt[1] = clock64();
            mark(2);
            while (true) {
                uint32_t stale = 0;
                for (uint32_t m = pend; m; m &= m - 1) {
                    const int n = __ffs(m) - 1;
                    const u64* src = tw + n * CW + 2 * lane;
                    if ((uint32_t)(src[0] >> 32) == ep && (uint32_t)(src[1] >> 32) == ep) {
                        *reinterpret_cast<float2*>(xs + n * KP + warp * CW + 2 * lane) =
                            make_float2(__uint_as_float((uint32_t)src[0]), __uint_as_float((uint32_t)src[1]));
                        pend &= ~(1u << n);
                    } else {
                        const uint32_t hx = ent[n * sz + 3 + 2 * side];
                        cp_async16(tw + n * CW + 2 * lane, HX + (int64_t)hx * H + cs + 2 * lane, 16u);
                        stale = 1;
                    }
                }
                XST(stF && rounds == 0, 19);
                XST(stF && rounds == 0, 20);
                if (!__any_sync(FULLMASK, stale)) break;
                ++rounds;
                cp_async_wait_all();
            }
            __syncwarp();
        } else if (op == INT_F || is_head) {
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
                    cin_ld2(cin + tid * CINMAX, pool + e[2] + H + lc * UM + uu, pool + e[4] + H + lc * UM + uu);
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
                cin_ld2(cin + tid * CINMAX, pool + e[2] + H + lc * UM + uu, pool + e[4] + H + lc * UM + uu);
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
                rv[0] = RV_LD(pool + e[1] + H + jj);
#pragma unroll
                for (int k = 0; k < 6; ++k) rv[1 + k] = RV_LD(pool + e[0] + (k + 1) * H + jj);
                rv[7] = RV_LD(pool + e[5] + H + jj);
                rv[8] = RV_LD(pool + e[7] + H + jj);
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
            // ---- forward of internal cells: matvec from registers (L123), NN in {4, 2, 1} nodes at a time.
            //      Each lane forms 8 NN partial gate sums (NN nodes x 4 rows x its unit pair) over its CPL
            //      columns; the 4 column-group lanes reduce them with a transposed halving (each lane keeps a
            //      quarter), the 8 warps' column slices meet in shared memory, and thread (node, unit) sums
            //      them and updates the cell ----
            auto fwd_group = [&](auto nnc, int n0) {
                constexpr int NN = decltype(nnc)::value;
                constexpr int V = NN * 8;
                XST(stF, 0);
                float2 a[NN][4];
#pragma unroll
                for (int n = 0; n < NN; ++n)
#pragma unroll
                    for (int r = 0; r < 4; ++r) a[n][r] = make_float2(0.f, 0.f);
#pragma unroll
                for (int t = 0; t < NG; ++t)
#pragma unroll
                    for (int n = 0; n < NN; ++n) {
                        const float4 x4 = *reinterpret_cast<const float4*>(xs + (n0 + n) * KP + warp * CW + 16 * t + 4 * cg);
                        const float xv[4] = {x4.x, x4.y, x4.z, x4.w};
#pragma unroll
                        for (int q = 0; q < 4; ++q)
#pragma unroll
                            for (int r = 0; r < 4; ++r)
                                a[n][r] = __ffma2_rn(wp[r][4 * t + q], make_float2(xv[q], xv[q]), a[n][r]);
                    }
                XST(stF, 1);
                // value v = (n * 4 + r) * 2 + unit; halving over lane bit 0, then bit 1
                float val[V];
#pragma unroll
                for (int n = 0; n < NN; ++n)
#pragma unroll
                    for (int r = 0; r < 4; ++r) { val[(n * 4 + r) * 2] = a[n][r].x; val[(n * 4 + r) * 2 + 1] = a[n][r].y; }
                const bool c0 = lane & 1, c1 = lane & 2;
#pragma unroll
                for (int i = 0; i < V / 2; ++i) {
                    const float snd = c0 ? val[i] : val[i + V / 2];
                    const float kp = c0 ? val[i + V / 2] : val[i];
                    val[i] = kp + __shfl_xor_sync(FULLMASK, snd, 1);
                }
#pragma unroll
                for (int i = 0; i < V / 4; ++i) {
                    const float snd = c1 ? val[i] : val[i + V / 4];
                    const float kp = c1 ? val[i + V / 4] : val[i];
                    val[i] = kp + __shfl_xor_sync(FULLMASK, snd, 2);
                }
                // kept value i is v = i + (2 c0 + c1) V / 4: node v / 8, row (v / 2) % 4, unit v % 2
                float* fb = fpb + fbuf * T::FPB + warp * (4 * UM * 4);
                const int vb = ((c0 ? 2 : 0) + (c1 ? 1 : 0)) * (V / 4);
                if constexpr (NN == 4) {
                    float* d = fb + (vb / 8) * (UM * 4) + 2 * ug * 4;
                    *reinterpret_cast<float4*>(d) = make_float4(val[0], val[2], val[4], val[6]);
                    *reinterpret_cast<float4*>(d + 4) = make_float4(val[1], val[3], val[5], val[7]);
                } else {
#pragma unroll
                    for (int i = 0; i < V / 4; ++i) {
                        const int v = vb + i;
                        fb[(v / 8) * (UM * 4) + (2 * ug + (v & 1)) * 4 + ((v >> 1) & 3)] = val[i];
                    }
                }
                __syncthreads();
                XST(stF, 2);
                if (tid < NN * UM) {
                    const int n = n0 + tid / UM, uu = tid % UM;
                    if (n < nb) {
                        const float* fs = fpb + fbuf * T::FPB + ((tid / UM) * UM + uu) * 4;
                        float gi = 0.f, go = 0.f, gu = 0.f, gfl = 0.f, gfr = 0.f;
#pragma unroll
                        for (int w = 0; w < NW; ++w) {
                            const float4 p4 = *reinterpret_cast<const float4*>(fs + w * (4 * UM * 4));
                            gi += p4.x; go += p4.y; gu += p4.z;
                            if (w < NW / 2) gfl += p4.w; else gfr += p4.w;
                        }
                        const uint32_t* e = ent + n * sz;
                        const uint32_t rec = e[0];
                        const int j = lc * UM + uu;
                        const float* b = bias + uu * 4;
                        const float* cv = cin + (n * UM + uu) * CINMAX;
                        const float i = fsigm(gi + b[0]), o = fsigm(go + b[1]), uv = ftanh(gu + b[2]);
                        const float fl = fsigm(gfl + b[3]), fr = fsigm(gfr + b[3]);
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
                }
                fbuf ^= 1;
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
            // columns.  Lane (ug, cg) of warp w forms the sums of its unit pair over its CPL columns (FFMA2 over
            // the pair, then the two halves added); the 8 unit-pair lanes of a column group reduce them with a
            // transposed halving (lane bits 2, 3, 4), so each lane ends with CPL / 8 adjacent columns summed
            // over all UM units of the CTA and publishes them as tagged PART slots: no shared memory and no
            // barrier between the products and the publish.
            if (kindB) {
                const bool b2 = lane & 4, b3 = lane & 8, b4 = lane & 16;
                // NP nodes at a time (independent product and shuffle chains interleave)
                auto tmv = [&](auto npc, int n0) {
                    constexpr int NP = decltype(npc)::value;
                    float dv[NP][CPL];
#pragma unroll
                    for (int p = 0; p < NP; ++p) {
                        const int n = n0 + p;
                        float2 gp[4];
#pragma unroll
                        for (int r = 0; r < 3; ++r) gp[r] = *reinterpret_cast<const float2*>(cin + (n * 5 + r) * UM + 2 * ug);
                        gp[3] = *reinterpret_cast<const float2*>(cin + (n * 5 + 3 + side) * UM + 2 * ug);
#pragma unroll
                        for (int k = 0; k < CPL; ++k) {
                            float2 d = __ffma2_rn(wp[0][k], gp[0], make_float2(0.f, 0.f));
                            d = __ffma2_rn(wp[1][k], gp[1], d);
                            d = __ffma2_rn(wp[2][k], gp[2], d);
                            d = __ffma2_rn(wp[3][k], gp[3], d);
                            dv[p][k] = d.x + d.y;
                        }
                    }
                    // halving over lane bits 2, 3, 4: kept value i is column index
                    // k = i + b2 CPL / 2 + b3 CPL / 4 + b4 CPL / 8 of the lane's CPL (k = 4 t + q)
#pragma unroll
                    for (int i = 0; i < CPL / 2; ++i)
#pragma unroll
                        for (int p = 0; p < NP; ++p) {
                            const float snd = b2 ? dv[p][i] : dv[p][i + CPL / 2];
                            const float kp = b2 ? dv[p][i + CPL / 2] : dv[p][i];
                            dv[p][i] = kp + __shfl_xor_sync(FULLMASK, snd, 4);
                        }
#pragma unroll
                    for (int i = 0; i < CPL / 4; ++i)
#pragma unroll
                        for (int p = 0; p < NP; ++p) {
                            const float snd = b3 ? dv[p][i] : dv[p][i + CPL / 4];
                            const float kp = b3 ? dv[p][i + CPL / 4] : dv[p][i];
                            dv[p][i] = kp + __shfl_xor_sync(FULLMASK, snd, 8);
                        }
#pragma unroll
                    for (int i = 0; i < CPL / 8; ++i)
#pragma unroll
                        for (int p = 0; p < NP; ++p) {
                            const float snd = b4 ? dv[p][i] : dv[p][i + CPL / 8];
                            const float kp = b4 ? dv[p][i + CPL / 8] : dv[p][i];
                            dv[p][i] = kp + __shfl_xor_sync(FULLMASK, snd, 16);
                        }
                    const int k0 = (b2 ? CPL / 2 : 0) + (b3 ? CPL / 4 : 0) + (b4 ? CPL / 8 : 0);
                    // column c: child side = c / H, unit jj = c % H, owner CTA m = jj / U, slot jj % U
                    const int c = warp * CW + 16 * (k0 / 4) + 4 * cg + (k0 % 4);
                    const int jj = c - side * H, m = jj / UM;
#pragma unroll
                    for (int p = 0; p < NP; ++p) {
                        const uint32_t pp = ent[(n0 + p) * sz + 4];
                        u64* dst = PART + ((((int64_t)pp * NCL + m) * NCL + lc) * 2 + side) * UM + (jj - m * UM);
                        if constexpr (CPL / 8 == 2) st_tag2(dst, dv[p][0], dv[p][1], ep);
                        else st_tag(dst, dv[p][0], ep);
                    }
                };
                int n0 = 0;
                for (; n0 + VPPS_DF_NP <= nb; n0 += VPPS_DF_NP) tmv(std::integral_constant<int, VPPS_DF_NP>{}, n0);
                for (; n0 < nb; ++n0) tmv(std::integral_constant<int, 1>{}, n0);
                XST(stB, 7);
                XST(stB, 8);
                XST(stB, 9);
                XST(stB, 10);
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
    // (every thread's writes, then the CTA barrier, then one GPU-scope fence and a release add by thread 0:
    //  the barrier orders the other threads' writes before thread 0's fence, whose cumulativity carries
    //  them to a grid that acquires the counter)
    if (P.done) {
        __syncthreads();
        if (tid == 0) {
            __threadfence();
            asm volatile("red.release.gpu.global.add.s32 [%0], 1;" ::"l"(P.done + grp) : "memory");
        }
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

int df_block(const void*) { return dev::df::DCfg<256, 256>::NTH; }

const Variant* df_variants(int32_t* n) {
    *n = (int32_t)(sizeof(kDfVariants) / sizeof(kDfVariants[0]));
    return kDfVariants;
}

}  // namespace vpps
