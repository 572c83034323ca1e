// VPPS recurrence of LSTM chains (sm_100a): the LSTM LM (M1, config 3) and the BiLSTM tagger (M2, config 4)
// with the recurrent matrix U held in registers across a group of co-resident CTAs (weight
// rows dealt to the register files, "the loaded weights ... reused by all the nodes that use the same
// weight matrix"), whole sentences per group (SPEC S5g's whole-graph groups, here per chain direction), and
// the signal/wait of L165 replaced by epoch-tagged 64-bit slots (as vpps_df):
//   HX[d][pos][H]               h of a position, read by every CTA of the group at the next step
//   PART[d][pos][m][k][UM]      CTA k's part of the transposed product Uᵀγ (L94, fn4) for the UM units CTA m
//                               owns, consumed by position pos (the previous step of the same chain)
// The input projections W x (all positions, one GEMM), the head and the weight gradients are dense
// products of the level path; this file replaces its per-time-step recurrent products:
//   forward   a_t = P[pos] + b + U h_{t-1};  i, f, o = σ, g = tanh;  c_t = f c_{t-1} + i g;  h_t = o tanh c_t
//   backward  ĉ = dc + dh o (1 - tanh² c);  γ = [ĉ g i(1-i); ĉ c_{t-1} f(1-f); dh tanh c o(1-o); ĉ i(1-g²)]
//             dc_{t-1} = ĉ f;  dh_{t-1} += Uᵀ γ   (dh = the head's dh + the successor's Uᵀ γ)
// Layout: group CTA lc owns hidden units lc·UM .. +UM-1 (all four gate rows); thread (u, τ) holds columns
// CG (τ + TU t) + q of those rows (128 registers at H = 128 / 256 / 512).
#include <cstdint>
#include <cuda_runtime.h>

#include "dev_common.cuh"
#include "vpps_kernel.cuh"

namespace vpps {
namespace dev {
namespace ch {

constexpr int NTH = 256;
constexpr int NB = 16;          // sentences per batch (a group's active sentences of a step, in slices)
constexpr int MAXS = 64;        // sentences per group
constexpr int NC = 2;           // sentences per transposed-product chunk (two alternating buffers)
typedef unsigned long long u64;

constexpr int ilog2(int x) { return x <= 1 ? 0 : 1 + ilog2(x / 2); }

template <int H>
struct Cfg {
    static constexpr int NCL = (4 * H * H + NTH * 128 - 1) / (NTH * 128);   // CTAs per group
    static constexpr int UM = H / NCL;                                       // units per CTA
    static constexpr int TU = NTH / UM;                                      // threads per unit
    static constexpr int CPT = H / TU;                                       // columns per thread
    static constexpr int CG = CPT >= 4 ? 4 : CPT;
    static constexpr int NG = CPT / CG;                                      // granules per thread
    static constexpr int WU = 32 / TU;                                       // units per warp
    // columns a lane keeps after the in-warp unit reduction (halving down to one granule, then butterflies)
    static constexpr int KEEP = CPT / WU >= CG ? CPT / WU : CG;
    static constexpr int LV = ilog2(WU);                 // exchange levels
    static constexpr int HL = ilog2(CPT / KEEP);         // of which halving
    static_assert(H % NCL == 0 && UM * TU == NTH && TU <= 32 && 32 % TU == 0 && CPT % CG == 0, "layout");
    static_assert(KEEP % CG == 0, "whole granules");
    static_assert(UM % 4 == 0, "PART slots in 16-byte pieces");
};

__device__ __forceinline__ u64 tagv(float v, uint32_t e) { return ((u64)e << 32) | __float_as_uint(v); }
__device__ __forceinline__ void st_tag(u64* p, float v, uint32_t e) {
    asm volatile("st.relaxed.gpu.global.b64 [%0], %1;" ::"l"(p), "l"(tagv(v, e)) : "memory");
}
// four tagged slots in one 32-byte store (each 8-byte element single-copy atomic); p is 32-byte aligned
__device__ __forceinline__ void st_tag4(u64* p, const float* v, uint32_t e) {
    asm volatile("st.relaxed.gpu.global.v4.b64 [%0], {%1, %2, %3, %4};"
                 ::"l"(p), "l"(tagv(v[0], e)), "l"(tagv(v[1], e)), "l"(tagv(v[2], e)), "l"(tagv(v[3], e)) : "memory");
}
// polls of slots other CTAs write in this kernel: relaxed GPU-scope loads (single-copy atomic 8 / 16 bytes)
__device__ __forceinline__ u64 ld_slot(const u64* p) {
    u64 v;
    asm volatile("ld.relaxed.gpu.global.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void ld_slot2(const u64* p, u64& a, u64& b) {
    asm volatile("ld.relaxed.gpu.global.v2.b64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}

// sentence table (host: tagger.cpp): [G, pre_0 .. pre_G, (off, len) x n]; group g's sentences are entries
// pre_g .. pre_{g+1}-1, longest first; position of step t: off + t (forward), off + len - 1 - t (backward
// direction of the tagger), its predecessor pos - dp... (dp = -1 forward, +1 backward)
__device__ __forceinline__ int pos_of(uint32_t off, uint32_t len, int t, int d) {
    return d == 0 ? (int)off + t : (int)(off + len) - 1 - t;
}

template <int H, int NGT>
__device__ __forceinline__ void load_weights(const ChainParams& P, int d, int lc, float (&w)[NGT][Cfg<H>::CPT]) {
    using C = Cfg<H>;
    const int tid = threadIdx.x, u = tid / C::TU, tau = tid % C::TU, j = lc * C::UM + u;
    const float* U = d == 0 ? P.U0 : P.U1;
#pragma unroll
    for (int k = 0; k < NGT; ++k)
#pragma unroll
        for (int t = 0; t < C::NG; ++t) {
            const float* src = U + (int64_t)(k * H + j) * H + C::CG * (tau + C::TU * t);
            if constexpr (C::CG == 4) {
                const float4 v = __ldg(reinterpret_cast<const float4*>(src));
                w[k][4 * t] = v.x; w[k][4 * t + 1] = v.y; w[k][4 * t + 2] = v.z; w[k][4 * t + 3] = v.w;
            } else {
#pragma unroll
                for (int q = 0; q < C::CG; ++q) w[k][C::CG * t + q] = __ldg(src + q);
            }
        }
}

// ---- forward: every step of the group's sentences, in order.  CELL 0 = LSTM (gates i, f, o, g), 1 = GRU
//      (M5, reading R-34: gates r, z, n with the reset on U_n h + b_hn; h' = (1 - z) n + z h) ----
template <int H, int CELL>
__global__ void __launch_bounds__(NTH, 1) vpps_chain_fwd(const ChainParams P) {
    using C = Cfg<H>;
    constexpr int TU = C::TU, UM = C::UM, CG = C::CG, NG = C::NG;
    constexpr int NGT = CELL == 0 ? 4 : 3;               // gate rows per unit
    extern __shared__ __align__(16) float csm[];
    float* xs0 = csm;                                  // two staging buffers [NB][H]
    __shared__ uint32_t s_off[MAXS], s_len[MAXS];
    const int tid = threadIdx.x;
    const int grp = blockIdx.x / C::NCL, lc = blockIdx.x % C::NCL;
    const int u = tid / TU, tau = tid % TU, j = lc * UM + u;
    const uint32_t* T = P.table;
    const int G = (int)T[0];
    if (grp >= G) return;
    const int s0 = (int)T[1 + grp], s1 = (int)T[2 + grp], ns = s1 - s0;
    const int d = grp < P.groups_dir0 ? 0 : 1;
    const uint32_t ep = P.epoch;
    for (int i = tid; i < ns; i += NTH) { s_off[i] = T[G + 2 + 2 * (s0 + i)]; s_len[i] = T[G + 3 + 2 * (s0 + i)]; }
    float w[NGT][C::CPT];
    load_weights<H, NGT>(P, d, lc, w);
    float bias[4], bias_h[3];                              // LSTM b; GRU b_i, b_h
#pragma unroll
    for (int k = 0; k < NGT; ++k) bias[k] = __ldg((CELL == 1 || d == 0 ? P.b0 : P.b1) + k * H + j);
#pragma unroll
    for (int k = 0; k < 3; ++k) bias_h[k] = CELL == 1 ? __ldg(P.b1 + k * H + j) : 0.f;
    const float* Pin = d == 0 ? P.P0 : P.P1;
    float* Cd = d == 0 ? P.C0 : P.C1;
    float* Gd = d == 0 ? P.G0 : P.G1;
    u64* HX = P.hx + (int64_t)d * P.T * H;             // each direction has its own slots
    __syncthreads();
    const int L = ns > 0 ? (int)s_len[0] : 0;
    int buf = 0;
    for (int t = 0; t < L; ++t) {
        int nact = 0;
        while (nact < ns && (int)s_len[nact] > t) ++nact;       // sentences longer than t: a prefix
        for (int b0 = 0; b0 < nact; b0 += NB, buf ^= 1) {
            const int nb = min(NB, nact - b0);
            float* x = xs0 + buf * NB * H;
            // ---- stage h_{t-1} of the batch's sentences (tagged slots of the group's CTAs) ----
            if (t > 0) {
                constexpr int PPS = H / 2;                      // 16-byte pieces per sentence
                while (true) {
                    int stale = 0;
                    for (int q = tid; q < nb * PPS; q += NTH) {
                        const int n = q / PPS, pc = q - n * PPS;
                        const int pp = pos_of(s_off[b0 + n], s_len[b0 + n], t - 1, d);
                        u64 a, b;
                        ld_slot2(HX + (int64_t)pp * H + 2 * pc, a, b);
                        if ((uint32_t)(a >> 32) == ep && (uint32_t)(b >> 32) == ep)
                            *reinterpret_cast<float2*>(x + n * H + 2 * pc) =
                                make_float2(__uint_as_float((uint32_t)a), __uint_as_float((uint32_t)b));
                        else
                            ++stale;
                    }
                    if (__syncthreads_count(stale) == 0) break;
                }
            }
            // ---- U h_{t-1}: 4 sentences at a time; the TU lanes of a unit reduce with a butterfly ----
            for (int n0 = 0; n0 < nb; n0 += 4) {
                float s[4][NGT];
                if (t > 0) {
                    float2 a[4][NGT];
#pragma unroll
                    for (int n = 0; n < 4; ++n)
#pragma unroll
                        for (int k = 0; k < NGT; ++k) a[n][k] = make_float2(0.f, 0.f);
#pragma unroll
                    for (int g = 0; g < NG; ++g) {
                        const int col = CG * (tau + TU * g);
#pragma unroll
                        for (int n = 0; n < 4; ++n) {
                            if (n0 + n >= nb) break;
                            float xv[CG];
                            lds<CG>(x + (n0 + n) * H + col, xv);
#pragma unroll
                            for (int q = 0; q + 1 < CG; q += 2)
#pragma unroll
                                for (int k = 0; k < NGT; ++k)
                                    a[n][k] = __ffma2_rn(make_float2(w[k][CG * g + q], w[k][CG * g + q + 1]),
                                                         make_float2(xv[q], xv[q + 1]), a[n][k]);
                            if constexpr (CG == 1)
#pragma unroll
                                for (int k = 0; k < NGT; ++k) a[n][k].x = fmaf(w[k][g], xv[0], a[n][k].x);
                        }
                    }
#pragma unroll
                    for (int n = 0; n < 4; ++n)
#pragma unroll
                        for (int k = 0; k < NGT; ++k) {
                            float v = a[n][k].x + a[n][k].y;
#pragma unroll
                            for (int o = TU / 2; o >= 1; o >>= 1) v += __shfl_xor_sync(FULLMASK, v, o);
                            s[n][k] = v;
                        }
                } else {
#pragma unroll
                    for (int n = 0; n < 4; ++n)
#pragma unroll
                        for (int k = 0; k < NGT; ++k) s[n][k] = 0.f;
                }
                // ---- cell: lane τ < 4 of the unit updates sentence n0 + τ ----
                const int n = n0 + tau;
                if (tau < 4 && n < nb) {
                    float a4[NGT];
#pragma unroll
                    for (int k = 0; k < NGT; ++k) {
                        float v = s[0][k];
#pragma unroll
                        for (int m = 1; m < 4; ++m) v = tau == m ? s[m][k] : v;
                        a4[k] = v;
                    }
                    const int pos = pos_of(s_off[b0 + n], s_len[b0 + n], t, d);
                    const int ppos = pos_of(s_off[b0 + n], s_len[b0 + n], t - 1, d);
                    const float* pr = Pin + (int64_t)pos * NGT * H;
                    float h;
                    if constexpr (CELL == 0) {
                        const float ig = fsigm(a4[0] + __ldg(pr + j) + bias[0]);
                        const float fg = fsigm(a4[1] + __ldg(pr + H + j) + bias[1]);
                        const float og = fsigm(a4[2] + __ldg(pr + 2 * H + j) + bias[2]);
                        const float gg = ftanh(a4[3] + __ldg(pr + 3 * H + j) + bias[3]);
                        const float cp = t > 0 ? Cd[(int64_t)ppos * H + j] : 0.f;
                        const float c = fg * cp + ig * gg;
                        h = og * ftanh(c);
                        Cd[(int64_t)pos * H + j] = c;
                        float* gr = Gd + (int64_t)pos * 4 * H;
                        gr[j] = ig; gr[H + j] = fg; gr[2 * H + j] = og; gr[3 * H + j] = gg;
                    } else {
                        const float ahr = bias_h[0] + a4[0], ahz = bias_h[1] + a4[1], ahn = bias_h[2] + a4[2];
                        const float rg = fsigm(__ldg(pr + j) + bias[0] + ahr);
                        const float zg = fsigm(__ldg(pr + H + j) + bias[1] + ahz);
                        const float ng = ftanh(__ldg(pr + 2 * H + j) + bias[2] + rg * ahn);
                        const float hp = t > 0 ? P.HH[(int64_t)ppos * P.HW + j] : 0.f;
                        h = (1.f - zg) * ng + zg * hp;
                        float* gr = Gd + (int64_t)pos * 4 * H;
                        gr[j] = rg; gr[H + j] = zg; gr[2 * H + j] = ng; gr[3 * H + j] = ahn;
                    }
                    if (t + 1 < (int)s_len[b0 + n]) st_tag(HX + (int64_t)pos * H + j, h, ep);   // next step's input
                    P.HH[(int64_t)pos * P.HW + d * H + j] = h;
                }
            }
        }
    }
}

// ---- backward: every step of the group's sentences, last first ----
template <int H, int CELL>
__global__ void __launch_bounds__(NTH, 1) vpps_chain_bwd(const ChainParams P) {
    using C = Cfg<H>;
    constexpr int TU = C::TU, UM = C::UM, CG = C::CG, NCL = C::NCL, KEEP = C::KEEP;
    constexpr int NGT = CELL == 0 ? 4 : 3;
    constexpr int NW = NTH / 32;
    extern __shared__ __align__(16) float csm[];
    float* gam_s = csm;                                // [NB][4][UM] this step's γ of the CTA's units
    float* dcs = gam_s + NB * 4 * UM;                  // [MAXS][UM] carried to the previous step: the LSTM's
                                                       // dc_{t-1}, the GRU's direct term dh z of dh_{t-1}
    float* dxb0 = dcs + MAXS * UM;                     // [2][NW][NC][H] warp slices of Uᵀγ
    __shared__ uint32_t s_off[MAXS], s_len[MAXS];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int grp = blockIdx.x / NCL, lc = blockIdx.x % NCL;
    const int u = tid / TU, tau = tid % TU;
    const uint32_t* T = P.table;
    const int G = (int)T[0];
    if (grp >= G) return;
    const int s0 = (int)T[1 + grp], s1 = (int)T[2 + grp], ns = s1 - s0;
    const int d = grp < P.groups_dir0 ? 0 : 1;
    const uint32_t ep = P.epoch;
    for (int i = tid; i < ns; i += NTH) { s_off[i] = T[G + 2 + 2 * (s0 + i)]; s_len[i] = T[G + 3 + 2 * (s0 + i)]; }
    for (int i = tid; i < MAXS * UM; i += NTH) dcs[i] = 0.f;
    float w[NGT][C::CPT];
    load_weights<H, NGT>(P, d, lc, w);
    const float* Cd = d == 0 ? P.C0 : P.C1;
    const float* Gd = d == 0 ? P.G0 : P.G1;
    float* Gam = d == 0 ? P.Gam0 : P.Gam1;
    u64* PART = P.part + (int64_t)d * P.T * NCL * H;   // each direction has its own slots
    __syncthreads();
    const int L = ns > 0 ? (int)s_len[0] : 0;
    int cbuf = 0;
    for (int t = L - 1; t >= 0; --t) {
        int nact = 0;
        while (nact < ns && (int)s_len[nact] > t) ++nact;
        for (int b0 = 0; b0 < nact; b0 += NB) {
            const int nb = min(NB, nact - b0);
            // ---- dh (head + the successor's Uᵀγ parts), cell backward: thread (sentence n, unit uu) ----
            for (int q = tid; q < nb * UM; q += NTH) {
                const int n = q / UM, uu = q - n * UM, jj = lc * UM + uu, sn = b0 + n;
                const uint32_t off = s_off[sn], len = s_len[sn];
                const int pos = pos_of(off, len, t, d);
                float dh = P.dHH[(int64_t)pos * P.HW + d * H + jj];
                if (t + 1 < (int)len) {
                    const u64* src = PART + (((int64_t)pos * NCL + lc) * NCL) * UM + uu;
                    u64 v[NCL];
#pragma unroll
                    for (int k = 0; k < NCL; ++k) v[k] = ld_slot(src + k * UM);
                    while (true) {
                        bool st = false;
#pragma unroll
                        for (int k = 0; k < NCL; ++k)
                            if ((uint32_t)(v[k] >> 32) != ep) { st = true; v[k] = ld_slot(src + k * UM); }
                        if (!st) break;
                    }
#pragma unroll
                    for (int k = 0; k < NCL; ++k) dh += __uint_as_float((uint32_t)v[k]);
                }
                const float carry = t + 1 < (int)len ? dcs[sn * UM + uu] : 0.f;
                const float* gr = Gd + (int64_t)pos * 4 * H;
                if constexpr (CELL == 0) {
                    const float i = gr[jj], f = gr[H + jj], o = gr[2 * H + jj], g = gr[3 * H + jj];
                    const float c = Cd[(int64_t)pos * H + jj];
                    const float cp = t > 0 ? Cd[(int64_t)pos_of(off, len, t - 1, d) * H + jj] : 0.f;
                    const float tc = ftanh(c);
                    const float chat = carry + dh * o * (1.f - tc * tc);
                    const float gam[4] = {chat * g * i * (1.f - i), chat * cp * f * (1.f - f), dh * tc * o * (1.f - o),
                                          chat * i * (1.f - g * g)};
                    float* go = Gam + (int64_t)pos * 4 * H;
#pragma unroll
                    for (int k = 0; k < 4; ++k) {
                        go[k * H + jj] = gam[k];
                        gam_s[(n * 4 + k) * UM + uu] = gam[k];
                    }
                    dcs[sn * UM + uu] = chat * f;                  // dc of step t-1 (same thread next time)
                } else {
                    const float dht = dh + carry;
                    const float rg = gr[jj], zg = gr[H + jj], ng = gr[2 * H + jj], ahn = gr[3 * H + jj];
                    const float hp = t > 0 ? P.HH[(int64_t)pos_of(off, len, t - 1, d) * P.HW + jj] : 0.f;
                    const float dan = dht * (1.f - zg) * (1.f - ng * ng);
                    const float dar = dan * ahn * rg * (1.f - rg);
                    const float daz = dht * (hp - ng) * zg * (1.f - zg);
                    float* gx = P.Gam0 + (int64_t)pos * 3 * H;
                    float* gh = P.Gam1 + (int64_t)pos * 3 * H;
                    gx[jj] = dar; gx[H + jj] = daz; gx[2 * H + jj] = dan;
                    gh[jj] = dar; gh[H + jj] = daz; gh[2 * H + jj] = dan * rg;
                    gam_s[(n * 4 + 0) * UM + uu] = dar;
                    gam_s[(n * 4 + 1) * UM + uu] = daz;
                    gam_s[(n * 4 + 2) * UM + uu] = dan * rg;
                    dcs[sn * UM + uu] = dht * zg;                  // dh_{t-1} += dh z (same thread next time)
                }
            }
            __syncthreads();
            if (t == 0) continue;                              // no predecessor: no Uᵀγ
            // ---- Uᵀγ for step t-1: per sentence this CTA's part over all H columns; the WU units of a warp
            //      are summed by halving exchanges, the NW warp slices in shared memory, chunks of NC
            //      sentences alternating between two buffers ----
            for (int n0 = 0; n0 < nb; n0 += NC, cbuf ^= 1) {
                float* buf = dxb0 + cbuf * NW * NC * H;
#pragma unroll
                for (int dn = 0; dn < NC; ++dn) {
                    const int n = n0 + dn;
                    if (n >= nb) break;
                    float gr[NGT];
#pragma unroll
                    for (int k = 0; k < NGT; ++k) gr[k] = gam_s[(n * 4 + k) * UM + u];
                    float v[C::CPT];
#pragma unroll
                    for (int c = 0; c < C::CPT; c += 2) {
                        float2 a = __ffma2_rn(make_float2(w[0][c], w[0][c + 1]), make_float2(gr[0], gr[0]), make_float2(0.f, 0.f));
#pragma unroll
                        for (int k = 1; k < NGT; ++k)
                            a = __ffma2_rn(make_float2(w[k][c], w[k][c + 1]), make_float2(gr[k], gr[k]), a);
                        v[c] = a.x;
                        v[c + 1] = a.y;
                    }
                    // in-warp sum over the WU units at lane distances TU, 2 TU, ...: halving exchanges while a lane
                    // keeps at least one granule (the lane keeps the half of the logical index range selected by
                    // its lane bit, always in v[0 ..)), then butterflies (duplicates: only the lane with the bit
                    // clear stores).  The lane ends with the sums of logical indices lo .. lo + KEEP - 1.
                    int lo = 0;
                    bool store = true;
#pragma unroll
                    for (int l = 0; l < C::LV; ++l) {
                        const int s = TU << l;
                        const bool up = lane & s;
                        if (l < C::HL) {
                            const int hh = C::CPT >> (l + 1);
#pragma unroll
                            for (int i = 0; i < hh; ++i) {
                                const float send = up ? v[i] : v[hh + i];
                                const float keep = up ? v[hh + i] : v[i];
                                v[i] = keep + __shfl_xor_sync(FULLMASK, send, s);
                            }
                            if (up) lo += hh;
                        } else {
#pragma unroll
                            for (int i = 0; i < KEEP; ++i) v[i] += __shfl_xor_sync(FULLMASK, v[i], s);
                            if (up) store = false;
                        }
                    }
                    // indices lo .. lo + KEEP - 1 = granules lo / CG ..: column CG (τ + TU g) + q
                    float* drow = buf + (warp * NC + dn) * H;
#pragma unroll
                    for (int i = 0; i < KEEP; i += CG) {
                        if (!store) break;
                        const int g = (lo + i) / CG;
                        const int col = CG * (tau + TU * g);
                        if constexpr (CG == 4)
                            *reinterpret_cast<float4*>(drow + col) = make_float4(v[i], v[i + 1], v[i + 2], v[i + 3]);
                        else
#pragma unroll
                            for (int q = 0; q < CG; ++q) drow[col + q] = v[i + q];
                    }
                }
                __syncthreads();
                constexpr int Q4 = H / 4;
                for (int i = tid; i < NC * Q4; i += NTH) {
                    const int dn = i / Q4, c = (i - dn * Q4) * 4, n = n0 + dn;
                    if (n >= nb) continue;
                    float s4[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
                    for (int ww = 0; ww < NW; ++ww) {
                        const float4 x = *reinterpret_cast<const float4*>(buf + (ww * NC + dn) * H + c);
                        s4[0] += x.x; s4[1] += x.y; s4[2] += x.z; s4[3] += x.w;
                    }
                    const int sn = b0 + n;
                    const int pp = pos_of(s_off[sn], s_len[sn], t - 1, d);
                    const int m = c / UM;
                    st_tag4(PART + (((int64_t)pp * NCL + m) * NCL + lc) * UM + (c - m * UM), s4, ep);
                }
                // (the next chunk writes the other buffer; this one is rewritten after the next barrier)
            }
        }
    }
}

}  // namespace ch
}  // namespace dev

namespace dev {
namespace ch {
template <int H>
constexpr size_t fwd_smem() { return (size_t)2 * NB * H * sizeof(float); }
template <int H>
constexpr size_t bwd_smem() {
    return ((size_t)NB * 4 * Cfg<H>::UM + (size_t)MAXS * Cfg<H>::UM + (size_t)2 * (NTH / 32) * NC * H) * sizeof(float);
}
}  // namespace ch
}  // namespace dev

#define VPPS_CHAIN_CASE(HH)                                                                          \
    case HH:                                                                                         \
        fwd = gru ? (const void*)&dev::ch::vpps_chain_fwd<HH, 1> : (const void*)&dev::ch::vpps_chain_fwd<HH, 0>; \
        bwd = gru ? (const void*)&dev::ch::vpps_chain_bwd<HH, 1> : (const void*)&dev::ch::vpps_chain_bwd<HH, 0>; \
        ncl = dev::ch::Cfg<HH>::NCL;                                                                 \
        sm_f = dev::ch::fwd_smem<HH>();                                                              \
        sm_b = dev::ch::bwd_smem<HH>();                                                              \
        break;

// CTAs per group of the register-resident recurrence at hidden size H (0: no specialisation)
int32_t chain_group_ctas(int32_t H) {
    switch (H) {
        case 32: return dev::ch::Cfg<32>::NCL;
        case 64: return dev::ch::Cfg<64>::NCL;
        case 128: return dev::ch::Cfg<128>::NCL;
        case 256: return dev::ch::Cfg<256>::NCL;
        case 512: return dev::ch::Cfg<512>::NCL;
        default: return 0;
    }
}

cudaError_t launch_chain(const ChainParams& P, int32_t H, int32_t n_groups, bool backward, cudaStream_t s, bool gru) {
    const void* fwd = nullptr;
    const void* bwd = nullptr;
    int ncl = 0;
    size_t sm_f = 0, sm_b = 0;
    switch (H) {
        VPPS_CHAIN_CASE(32)
        VPPS_CHAIN_CASE(64)
        VPPS_CHAIN_CASE(128)
        VPPS_CHAIN_CASE(256)
        VPPS_CHAIN_CASE(512)
        default: return cudaErrorInvalidValue;
    }
    const void* fn = backward ? bwd : fwd;
    const size_t smem = backward ? sm_b : sm_f;
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    ChainParams p = P;
    void* args[] = {&p};
    // cooperative: the CTAs of a group poll each other's slots, so all of them must be resident
    return cudaLaunchCooperativeKernel(fn, dim3(n_groups * ncl), dim3(dev::ch::NTH), args, smem, s);
}

}  // namespace vpps
