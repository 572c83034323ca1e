// Weight gradients of the binary Tree-LSTM's dataflow path on the tensor cores ("concatenate all
// the left hand side and all the right hand side tensors that participate in the outer-product for each
// weight matrix, and use dense matrix-matrix multiplication"), per replica group as soon as the group's 16
// vpps_df CTAs have counted themselves done (the work fills the SMs of finished groups while the slowest
// group still runs; L185's one GEMM per matrix becomes one GEMM per matrix and group, summed in grads):
//   p0  dU_iou [3H x 2H] = Σ_int  g_iou [h_l; h_r]ᵀ     A(m, k) = pool[rec_k + 7H + m], B(k, n) = h_l / h_r of k
//   p1  dU_fl  [H x H]   = Σ_int  g_fl h_lᵀ             A = pool[rec_k + 10H + m],      B = pool[rec_l(k) + n]
//   p2  dU_fr  [H x H]   = Σ_int  g_fr h_rᵀ             A = pool[rec_k + 11H + m],      B = pool[rec_r(k) + n]
//   p3  dW_iou [3H x E]  = Σ_leaf g x_tokᵀ              A = pool[rec_k + 5H + m],       B = inputs[tok_k E + n]
//   p4  dX[tok_m] += g_leaf(m)ᵀ W_iou  [leaves x E]     A(m, k) = pool[rec_m + 5H + k], B(k, n) = W_iou[k E + n]
// Operands are gathered row by row through the group's node lists by 16-byte cp.async into a raw ring two
// chunks deep, then split into tc_common.cuh's 128 x 128 3xTF32 stages.  Work items = (group, product,
// 128 x 128 tile, K range); persistent CTAs claim the items of finished groups; partial tiles are added into
// grads / dX (cleared by the leaf kernel) with red.global.add.v4.  Once every item is counted the CTAs apply
// the SGD update (L129, L197) and one CTA copies the summed loss to mapped host memory.
#include <algorithm>
#include <atomic>
#include <cstdint>
#include <cuda_runtime.h>

#include "dev_common.cuh"
#include "tc_common.cuh"
#include "vpps_kernel.cuh"

namespace vpps {
namespace dev {
namespace dwtc {
using namespace tcc;

constexpr int NP = 5;

constexpr int MAXG = 16;

struct Params {
    const float* pool;
    const float* inputs;
    const float* w_iou;
    float* grads;
    float* d_inputs;                 // dX or nullptr (p4 skipped)
    const uint32_t* ints;            // n_int x (rec, rec_l, rec_r), grouped by replica group
    const uint32_t* leaves;          // n_leaf x (rec, token), grouped by replica group
    int32_t H, E;
    int64_t off[8];
    int32_t ksplit[NP];              // K per item (p0-p3: whole group lists up to KMAXI; p4: slices of 3H)
    int32_t n_grp;
    int32_t grp[MAXG];               // groups in claiming order (expected to finish first go first)
    int32_t int_off[MAXG + 1], leaf_off[MAXG + 1];
    int32_t gfirst[MAXG][NP + 1];    // item prefix over the products of each group
    const int32_t* done;             // per-group completion counters (vpps_df)
    int32_t* claim;                  // per-group claim counters (zeroed per pass)
    int32_t done_target;
    int32_t total;
    // tail
    int32_t* fin;
    int32_t* tail_claim;
    int32_t mode;
    float* params;
    int64_t n_floats;
    float lr, wd;
    const float* loss_src;
    float* loss_dst;
};

__host__ __device__ inline void product_shape(int p, int H, int E, int n_int, int n_leaf, bool dx, int& M, int& N,
                                              int& K) {
    switch (p) {
        case 0: M = 3 * H; N = 2 * H; K = n_int; break;
        case 1:
        case 2: M = H; N = H; K = n_int; break;
        case 3: M = 3 * H; N = E; K = n_leaf; break;
        default: M = n_leaf; N = E; K = dx ? 3 * H : 0;
    }
    if (M <= 0 || K <= 0) M = K = 0;
}

// Staging: the operands are gathered node by node, so each chunk is first copied with 16-byte cp.async into
// a raw shared-memory ring (two chunks ahead: no registers held across the L2 round trip) and then converted
// into the canonical hi / lo stage of the tensor core.  Raw layouts: an operand contiguous along its rows
// (every A but p4's, every B) as [32 k][RS] with RS = 132 (the conversion reads one k per lane: rows 132
// floats apart hit distinct banks); p4's A (contiguous along k) as [128 rows][32 k].
constexpr int RS = BM + 4;
constexpr int RAW_F = BKC * RS;                 // floats of one raw operand chunk (>= 128 x 32)
constexpr int KMAXI = 1024;                     // node offsets staged per item (host keeps K per item below)
constexpr size_t SMEM_DW = tcc::SMEM + (size_t)2 * 2 * RAW_F * sizeof(float);

// per-item operand offsets (floats, shared memory): element A(m, k) = abase + aoff[k] + m (p4: aoff[m] + k),
// B(k, n) = bbase + boff[k] + n
__device__ __forceinline__ void copy_chunk(const float* abase, const float* bbase, const uint32_t* aoff,
                                           const uint32_t* boff, bool a_kc, int m0, int M, int n0, int N, int kc0,
                                           int kb, int ke, float* rawA, float* rawB) {
    const int tid = threadIdx.x;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int g = tid + NT * q;
        if (a_kc) {                                    // [128 rows][32 k]: row g / 8, k 4 (g % 8)
            const int r = g / 8, k = 4 * (g % 8), gr = m0 + r, gk = kc0 + k;
            const bool ok = gr < M && gk < ke;
            const float* src = ok ? abase + aoff[r] + gk : abase;
            cp_async16(rawA + r * BKC + k, src, ok ? (gk + 3 < ke ? 16u : 4u * (ke - gk)) : 0u);
        } else {                                       // [32 k][RS]: k g / 32, rows 4 (g % 32)
            const int k = g / 32, r = 4 * (g % 32), gr = m0 + r, gk = kc0 + k;
            const bool ok = gk < ke && gr < M;         // (M is a multiple of 4 here)
            const float* src = ok ? abase + aoff[gk - kb] + gr : abase;
            cp_async16(rawA + k * RS + r, src, ok ? 16u : 0u);
        }
        {
            const int k = g / 32, r = 4 * (g % 32), gn = n0 + r, gk = kc0 + k;
            const bool ok = gk < ke && gn < N;
            const float* src = ok ? bbase + boff[gk - kb] + gn : bbase;
            cp_async16(rawB + k * RS + r, src, ok ? 16u : 0u);
        }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
}

// raw chunk -> canonical hi / lo copies (the layout of tc_common.cuh)
__device__ __forceinline__ void convert_rows(const float* raw, float* hi, float* lo) {
    // row-contiguous raw [32 k][RS]: lane = k, piece = rows 4 (g / 32) .. +3 (transposing 4-byte stores)
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int g = threadIdx.x + NT * q, k = g % 32, r0 = 4 * (g / 32);
        const float4 v = *reinterpret_cast<const float4*>(raw + k * RS + r0);
        const float e[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
        for (int t = 0; t < 4; ++t) {
            const int r = r0 + t;
            const int o = (k >> 2) * (LBO / 4) + (r >> 3) * 32 + (r & 7) * 4 + (k & 3);
            const float h = tf32_hi(e[t]);
            hi[o] = h;
            lo[o] = e[t] - h;
        }
    }
}
__device__ __forceinline__ void convert_kc(const float* raw, float* hi, float* lo) {
    // k-contiguous raw [128 rows][32 k]: piece = row g / 8, k 4 (g % 8) .. +3 (16-byte stores)
#pragma unroll
    for (int q = 0; q < 4; ++q) {
        const int g = threadIdx.x + NT * q, r = g / 8, k4 = g % 8;
        const float4 v = *reinterpret_cast<const float4*>(raw + r * BKC + 4 * k4);
        const int o = k4 * (LBO / 4) + (r >> 3) * 32 + (r & 7) * 4;
        const float4 h = make_float4(tf32_hi(v.x), tf32_hi(v.y), tf32_hi(v.z), tf32_hi(v.w));
        *reinterpret_cast<float4*>(hi + o) = h;
        *reinterpret_cast<float4*>(lo + o) = make_float4(v.x - h.x, v.y - h.y, v.z - h.z, v.w - h.w);
    }
}

__global__ void __launch_bounds__(NT, 1) vpps_dw_tc(const Params P) {
    extern __shared__ __align__(128) float tsm[];
    __shared__ uint32_t tmem_base;
    __shared__ __align__(8) uint64_t mbar[2];
    __shared__ int pick[3];
    __shared__ uint32_t aoff[KMAXI], boff[KMAXI];
    float* canon = reinterpret_cast<float*>((reinterpret_cast<uintptr_t>(tsm) + 127) & ~uintptr_t(127));
    float* raw = canon + 2 * STAGE_F;                 // 2 stages x (A, B)
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int H = P.H;
    setup(&tmem_base, mbar);
    const uint32_t tmem = tmem_base;
    uint32_t phases = 0u;
    while (true) {
        // claim an item of a group whose CTAs have all counted themselves done (lane q looks at group grp[q])
        if (tid < 32) {
            const int g = lane < P.n_grp ? P.grp[lane] : -1;
            uint32_t c = 0, d = 0;
            if (g >= 0) {
                asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(c) : "l"(P.claim + g) : "memory");
                asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(d) : "l"(P.done + g) : "memory");
            }
            const int items = g >= 0 ? P.gfirst[g][NP] : 0;
            const bool left = g >= 0 && (int)c < items;
            unsigned ready = __ballot_sync(0xffffffffu, left && (int)d >= P.done_target);
            int got_g = -1, got_i = -1;
            while (ready && got_g < 0) {
                const int q = __ffs(ready) - 1;
                int i = 0;
                if (lane == q) i = atomicAdd(P.claim + g, 1);
                i = __shfl_sync(0xffffffffu, i, q);
                const int gq = __shfl_sync(0xffffffffu, g, q);
                if (i < P.gfirst[gq][NP]) { got_g = gq; got_i = i; }
                ready &= ready - 1;
            }
            const unsigned any_left = __ballot_sync(0xffffffffu, left);
            if (lane == 0) { pick[0] = got_g; pick[1] = got_i; pick[2] = any_left != 0; }
        }
        __syncthreads();
        const int g = pick[0], it = pick[1], rem = pick[2];
        __syncthreads();
        if (g < 0) {
            if (!rem) break;
            __nanosleep(256);
            continue;
        }
        const int n_int = P.int_off[g + 1] - P.int_off[g], n_leaf = P.leaf_off[g + 1] - P.leaf_off[g];
        const uint32_t* ints = P.ints + 3 * P.int_off[g];
        const uint32_t* leaves = P.leaves + 2 * P.leaf_off[g];
        int p = 0;
        while (it >= P.gfirst[g][p + 1]) ++p;
        int M, N, K;
        product_shape(p, H, P.E, n_int, n_leaf, P.d_inputs != nullptr, M, N, K);
        const int local = it - P.gfirst[g][p];
        const int tn = (N + BN - 1) / BN, per_split = ((M + BM - 1) / BM) * tn;
        const int sp = local / per_split, t = local - sp * per_split;
        const int m0 = (t / tn) * BM, n0 = (t % tn) * BN;
        const int kb = sp * P.ksplit[p], ke = min(K, kb + P.ksplit[p]);
        const int nch = (ke - kb + BKC - 1) / BKC;
        const bool a_kc = p == 4;
        // operand offsets of the item (node lists, PAPER L185's concatenated operands)
        const float* abase = P.pool;
        const float* bbase = p == 3 ? P.inputs : (p == 4 ? P.w_iou : P.pool);
        if (a_kc) {
            for (int r = tid; r < BM; r += NT) aoff[r] = m0 + r < M ? __ldcg(leaves + (2 * (m0 + r))) + 5 * H : 0u;
            for (int k = tid; k < ke - kb; k += NT) boff[k] = (uint32_t)(kb + k) * (uint32_t)P.E;
        } else {
            for (int k = tid; k < ke - kb; k += NT) {
                const int node = kb + k;
                if (p == 3) {
                    aoff[k] = __ldcg(leaves + (2 * node)) + 5 * H;
                    boff[k] = __ldcg(leaves + (2 * node + 1)) * (uint32_t)P.E;
                } else {
                    const uint32_t rec = __ldcg(ints + (3 * node));
                    aoff[k] = rec + (p == 0 ? 7 : (p == 1 ? 10 : 11)) * H;
                    boff[k] = p == 1 || (p == 0 && n0 < H) ? __ldcg(ints + (3 * node + 1))
                                                           : __ldcg(ints + (3 * node + 2)) - (p == 0 ? H : 0);
                }
            }
        }
        __syncthreads();
        // prologue: chunks 0 and 1 in flight
        for (int c = 0; c < 2; ++c) {
            if (c < nch)
                copy_chunk(abase, bbase, aoff, boff, a_kc, m0, M, n0, N, kb + c * BKC, kb, ke, raw + c * 2 * RAW_F,
                           raw + c * 2 * RAW_F + RAW_F);
            else asm volatile("cp.async.commit_group;" ::: "memory");
        }
        for (int c = 0; c < nch; ++c) {
            const int st = c & 1;
            float* rA = raw + st * 2 * RAW_F;
            float* Ah = canon + st * STAGE_F;
            asm volatile("cp.async.wait_group 1;" ::: "memory");      // this thread's copies of chunk c
            __syncthreads();                                           // ... and everyone else's
            if (c >= 2) { mbar_wait(smem_u32(&mbar[st]), (phases >> st) & 1u); phases ^= 1u << st; }
            if (a_kc) convert_kc(rA, Ah, Ah + OP_F);
            else convert_rows(rA, Ah, Ah + OP_F);
            convert_rows(rA + RAW_F, Ah + 2 * OP_F, Ah + 3 * OP_F);
            issue_chunk(tmem, Ah, &mbar[st], c == 0);                 // (its barrier also frees raw stage st)
            if (c + 2 < nch)
                copy_chunk(abase, bbase, aoff, boff, a_kc, m0, M, n0, N, kb + (c + 2) * BKC, kb, ke, rA, rA + RAW_F);
            else asm volatile("cp.async.commit_group;" ::: "memory");
        }
        // drain: the last commit covers every MMA of the item; both stages are then free for the next item
        if (nch > 0) {
            const int st = (nch - 1) & 1;
            mbar_wait(smem_u32(&mbar[st]), (phases >> st) & 1u);
            phases ^= 1u << st;
            if (nch >= 2) {                       // the other stage's last completion was not waited for
                const int so = st ^ 1;
                mbar_wait(smem_u32(&mbar[so]), (phases >> so) & 1u);
                phases ^= 1u << so;
            }
        }
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        if (nch > 0) {
            const int row = m0 + 32 * (warp & 3) + lane, cb = 64 * (warp >> 2);
            float* out = nullptr;
            if (row < M)
                out = p == 4 ? P.d_inputs + (int64_t)__ldcg(leaves + (2 * row + 1)) * P.E
                             : P.grads + P.off[p == 3 ? 0 : p + 1] + (int64_t)row * N;
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                uint32_t r[16];
                load16(tmem, cb + 16 * q, r);
                const int nb = n0 + cb + 16 * q;
                if (out) {
#pragma unroll
                    for (int j = 0; j < 16; j += 4)
                        if (nb + j < N) {     // N is a multiple of 4
                            const float v[4] = {__uint_as_float(r[j]), __uint_as_float(r[j + 1]),
                                                __uint_as_float(r[j + 2]), __uint_as_float(r[j + 3])};
                            red_add<4>(out + nb + j, v);
                        }
                }
            }
        }
        // every thread's TMEM reads (and the item's reductions) precede the next item's first MMA and the count
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncthreads();
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        if (tid == 0) asm volatile("red.release.gpu.global.add.s32 [%0], 1;" ::"l"(P.fin) : "memory");
    }
    teardown(tmem);
    // ---- tail: SGD over the flat parameters once every item is counted (L129, L197), loss read-back (L199) ----
    if (tid == 0) {
        uint32_t f;
        while (true) {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(f) : "l"(P.fin) : "memory");
            if ((int)f >= P.total) break;
            __nanosleep(64);
        }
    }
    __syncthreads();
    constexpr int CV = 4;
    constexpr int64_t CH = 4 * CV * NT;
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
            const int64_t k = tid + NT * q;
            if (k < n4) { a[q] = __ldcg(p4 + k); b[q] = __ldcg(g4 + k); }
        }
#pragma unroll
        for (int q = 0; q < CV; ++q) {
            const int64_t k = tid + NT * q;
            if (k >= n4) break;
            a[q].x -= lr * (b[q].x + wd * a[q].x); a[q].y -= lr * (b[q].y + wd * a[q].y);
            a[q].z -= lr * (b[q].z + wd * a[q].z); a[q].w -= lr * (b[q].w + wd * a[q].w);
            p4[k] = a[q];
        }
    }
}

}  // namespace dwtc
}  // namespace dev

// Host: per group and product the 128 x 128 tiles and K slices (p0-p3 take the group's whole node list up to
// KMAXI nodes per item; the leaf dX's K = 3H runs in slices of 192), groups in the claiming order.
bool launch_dw_tc(const float* pool, const float* inputs, float* d_inputs, float* params, float* grads,
                  const uint32_t* ints, const uint32_t* leaves, int32_t n_grp, const int32_t* int_off,
                  const int32_t* leaf_off, const int32_t* order, int32_t* done, int32_t done_target, int32_t H,
                  int32_t E, const int64_t* off, int64_t n_floats, int32_t mode, float lr, float wd, cudaStream_t s,
                  const float* loss_src, float* loss_dst, int32_t n_sm) {
    using namespace dev::dwtc;
    using dev::tcc::BM;
    using dev::tcc::BN;
    if ((H % 4) || (E % 4) || (n_floats % 4) || n_grp > MAXG || !done) return false;
    Params P{};
    P.pool = pool; P.inputs = inputs; P.w_iou = params + off[0]; P.grads = grads; P.d_inputs = d_inputs;
    P.ints = ints; P.leaves = leaves; P.H = H; P.E = E;
    for (int i = 0; i < 8; ++i) P.off[i] = off[i];
    for (int p = 0; p < NP; ++p) P.ksplit[p] = p == 4 ? 192 : KMAXI;
    P.n_grp = n_grp;
    int total = 0;
    for (int q = 0; q <= n_grp; ++q) { P.int_off[q] = int_off[q]; P.leaf_off[q] = leaf_off[q]; }
    for (int q = 0; q < n_grp; ++q) {
        const int g = order ? order[q] : q;
        P.grp[q] = g;
        const int ni = int_off[g + 1] - int_off[g], nl = leaf_off[g + 1] - leaf_off[g];
        P.gfirst[g][0] = 0;
        for (int p = 0; p < NP; ++p) {
            int M, N, K;
            product_shape(p, H, E, ni, nl, d_inputs != nullptr, M, N, K);
            const int items = M ? ((M + BM - 1) / BM) * ((N + BN - 1) / BN) * ((K + P.ksplit[p] - 1) / P.ksplit[p]) : 0;
            P.gfirst[g][p + 1] = P.gfirst[g][p] + items;
        }
        total += P.gfirst[g][NP];
    }
    P.total = total;
    P.done = done;
    P.claim = done + 16;
    P.fin = done + 32;
    P.tail_claim = done + 33;
    P.done_target = done_target;
    P.mode = mode; P.params = params; P.n_floats = n_floats; P.lr = lr; P.wd = wd;
    P.loss_src = loss_src; P.loss_dst = loss_dst;
    static std::atomic<uint64_t> attr_done{0};
    int dev = 0;
    cudaGetDevice(&dev);
    if (!(attr_done.load() >> (dev & 63) & 1)) {
        if (cudaFuncSetAttribute(vpps_dw_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM_DW) != cudaSuccess)
            return false;
        attr_done.fetch_or(uint64_t(1) << (dev & 63));
    }
    // persistent, one CTA per SM, programmatic dependent of vpps_df: CTAs become resident on the SMs the
    // finished groups release and claim those groups' items (no griddepcontrol.wait: the per-group counters
    // order the reads of each group's records)
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.gridDim = dim3(std::max(1, std::min(total, n_sm)));
    cfg.blockDim = dim3(dev::tcc::NT);
    cfg.dynamicSmemBytes = SMEM_DW;
    cfg.stream = s;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, vpps_dw_tc, P) == cudaSuccess;
}

}  // namespace vpps
