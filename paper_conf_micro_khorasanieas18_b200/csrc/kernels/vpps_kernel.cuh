// Kernel-side declarations shared by the launcher (api.cu) and the kernel translation unit.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace vpps {

struct KParams {
    float* params;          // DRAM master copy (flat, vpps_layout offsets)
    float* grads;           // gradient output (mode 0)
    const float* inputs;    // caller's input table [rows x E]
    float* d_inputs;        // gradient of the input table, or nullptr
    float* pool;            // activation pool (SPEC §S7)
    const uint32_t* script; // encoded script (SPEC §E)
    int64_t off[8];         // parameter offsets in floats
    int32_t n_g, n_act, C, mode;   // mode 0: write grads; 1: fused SGD update
    int32_t G;                     // replica groups (SPEC P1); G > 1 sums gradients across groups
    int64_t loss_word;
    float lr, wd;
    uint64_t* prof;         // optional globaltimer trace (vpps_set_profile_buffer), or nullptr
    int64_t prof_stride;
    int32_t* done;          // cluster path: per-group completion counters (one increment per CTA), or nullptr
};

// Dataflow kernel (vpps_dataflow.cu): groups of 16 co-resident CTAs, epoch-tagged cross-CTA slots.
struct DfParams {
    float* params;
    float* grads;
    float* pool;
    const uint32_t* script;     // device blob; the group programs start at df_off
    int64_t df_off;
    int64_t off[8];
    int32_t C;
    const uint32_t* epoch;      // device pass counter (advanced by the leaf kernel): tag of this pass's slots
    int64_t loss_word;
    int64_t df_hx, df_part, df_hd;   // word offsets of the tagged regions in the pool
    uint64_t* prof;
    int64_t prof_stride;
    int32_t* done;              // per-group completion counters, or nullptr
    int64_t pool_words, n_hx, n_part, n_hd;   // record region and slot counts (bounds of the checked build)
};

// Device allocations of library-owned buffers (include/vpps.h vpps_alloc_fn / vpps_free_fn): the caller's
// callbacks, or stream-ordered cudaMallocAsync / cudaFreeAsync when they are NULL.
struct DevAlloc {
    void* (*alloc_fn)(size_t bytes, void* stream, void* ctx) = nullptr;
    void (*free_fn)(void* p, void* stream, void* ctx) = nullptr;
    void* ctx = nullptr;
    void* get(size_t bytes, cudaStream_t s) const {
        if (alloc_fn) return alloc_fn(bytes, (void*)s, ctx);
        void* p = nullptr;
        return cudaMallocAsync(&p, bytes, s) == cudaSuccess ? p : nullptr;
    }
    void put(void* p, cudaStream_t s) const {
        if (!p) return;
        if (free_fn) free_fn(p, (void*)s, ctx);
        else cudaFreeAsync(p, s);
    }
};

struct Variant {
    int32_t cell, H, E, umax;
    const void* fn;
    size_t (*smem_bytes)(int32_t C);
};

// Table of compiled specialisations (vpps_kernel.cu).
const Variant* variants(int32_t* n);
// Cluster-replica specialisations (vpps_cluster.cu); Variant.umax holds the cluster size.
const Variant* cluster_variants(int32_t* n);
// Dataflow specialisations (vpps_dataflow.cu); Variant.umax holds the group size.
const Variant* df_variants(int32_t* n);
const void* df_prof_fn(const void* fn);   // the trace-enabled instantiation of a dataflow variant
int df_block(const void* fn);             // threads per CTA of a dataflow specialisation
const void* fb_prof_fn(const void* fn);   // ... of a grid-kernel variant
// dW = Σ g xᵀ per weight matrix from the recorded operands, fused SGD when mode == 1.
// Also forms the leaf input gradient dX[tok] += W_iouᵀ g_leaf when d_inputs is not null.  Node lists are
// grouped by replica group (offsets int_off / leaf_off, n_grp + 1 entries); with `early` the kernel is a
// programmatic dependent launch of vpps_cl / vpps_df; persistent CTAs claim a group's tiles (counters
// done[16 + group], zeroed per pass) once done[group] >= done_target.
void launch_dw_gemm(const float* pool, const float* inputs, float* d_inputs, float* params, float* grads,
                    const uint32_t* int_nodes, const uint32_t* leaf_nodes, int32_t n_grp, const int32_t* int_off,
                    const int32_t* leaf_off, const int32_t* order, int32_t* done, int32_t done_target,
                    bool early, int32_t H, int32_t E, const int64_t* off, int64_t n_floats, int32_t mode, float lr,
                    float wd, cudaStream_t s, uint64_t* trace = nullptr, const float* loss_src = nullptr,
                    float* loss_dst = nullptr);
// The dataflow path's weight gradients on the tensor cores (vpps_dwtc.cu): dU_iou, dU_fl, dU_fr, dW_iou and
// the leaf dX per replica group, claimed by persistent CTAs once done[group] >= done_target (programmatic
// dependent of vpps_df), 128 x 128 3xTF32 tiles; SGD (mode 1) and the loss copy in the tail.  Counters as for
// launch_dw_gemm (done, claim = done + 16, fin / tail = done + 32 / 33; zeroed per pass).
bool launch_dw_tc(const float* pool, const float* inputs, float* d_inputs, float* params, float* grads,
                  const uint32_t* ints, const uint32_t* leaves, int32_t n_grp, const int32_t* int_off,
                  const int32_t* leaf_off, const int32_t* order, int32_t* done, int32_t done_target, int32_t H,
                  int32_t E, const int64_t* off, int64_t n_floats, int32_t mode, float lr, float wd, cudaStream_t s,
                  const float* loss_src, float* loss_dst, int32_t n_sm);
// (with completion counters the kernel also applies the SGD update and copies *loss_src to loss_dst, a
//  device-visible pointer to mapped host memory, after the last item; otherwise separate launches do)
// Leaf level of the binary cell as one GEMM + fused cell (vpps_leaf.cu): records h, c, i, o, u of every
// leaf before the cluster kernel.
// It also zeroes up to 4 float ranges (zero_ptr[r], zero_n[r] floats, multiples of 4; nullptr = unused)
// and advances the device pass counter `epoch` (if not null): the per-pass clearing without memset calls.
void launch_leaf_fwd(const float* W, const float* b, const float* inputs, float* pool, const uint32_t* leaves,
                     int32_t n_leaf, int32_t H, int32_t E, float* const* zero_ptr, const int64_t* zero_n,
                     uint32_t* epoch, cudaStream_t s, const void* prefetch = nullptr, int64_t prefetch_bytes = 0,
                     int64_t n_rows = 0);   // n_rows > 0: rows of `inputs` (enables the TMA-fed variant)
// Per-device function attributes (dynamic shared memory) of the gradient GEMM and the leaf kernels.
cudaError_t setup_dw_gemm_attrs();
cudaError_t setup_leaf_attrs();
// Elementwise SGD on the flat buffer (K3): p -= lr * (g + wd * p).
void launch_sgd(float* p, const float* g, int64_t n, float lr, float wd, cudaStream_t s);
// Dense FP32 product of the level paths (vpps_gemm.cu): row-major C = op(A) op(B) + beta C (beta 0 or 1).
cudaError_t gemm_f32(cudaStream_t s, bool ta, bool tb, int M, int N, int K, const float* A, int lda, const float* B,
                     int ldb, float* C, int ldc, float beta);
// Register-resident recurrence of LSTM chains (vpps_chain.cu): groups of chain_group_ctas(H) co-resident
// CTAs hold U, whole sentences per group, epoch-tagged slots between the steps.  table (device): [G,
// pre_0 .. pre_G, (off, len) per sentence]; groups [0, groups_dir0) run direction 0, the rest direction 1.
struct ChainParams {
    const uint32_t* table;
    int32_t groups_dir0;
    int32_t HW;                      // row stride of HH / dHH (H, or 2H for the tagger)
    uint32_t epoch;                  // tag of this pass's slots (never 0)
    const float *U0, *U1, *b0, *b1;  // recurrent matrices and biases of the two directions (GRU: U0, b0 = b_i,
                                     // b1 = b_h; Gam0 = γ_x, Gam1 = γ_h; P0 is W x [T][3H])
    const float *P0, *P1;            // input projections W x [T][4H] (bias not included)
    float* HH;                       // h [T][HW] (direction d at column d H)
    float *C0, *C1, *G0, *G1;        // c [T][H], gates (i, f, o, g) [T][4H] per direction
    const float* dHH;                // the head's dh [T][HW]
    float *Gam0, *Gam1;              // γ [T][4H] per direction (left operands of the weight gradients)
    unsigned long long* hx;          // [dirs][T][H] tagged h slots
    unsigned long long* part;        // [dirs][T][NCL][NCL][UM] tagged Uᵀγ parts
    int64_t T;                       // positions
};
int32_t chain_group_ctas(int32_t H);
cudaError_t launch_chain(const ChainParams& P, int32_t H, int32_t n_groups, bool backward, cudaStream_t s,
                         bool gru = false);
// Level-synchronous path (vpps_level.cu): context (cuBLAS handle + work buffers) and one training pass.
void* level_ctx_create(const DevAlloc* alloc);
void level_ctx_destroy(void* ctx);
int level_pass(void* ctx, const float* params, const int64_t* off, float* grads, float* pool, const float* inputs,
               float* d_inputs, const uint32_t* d_blob, int64_t lv_int, int64_t lv_leaf, int64_t lv_head,
               const int32_t* lv_start, int32_t L, int64_t n_int, int64_t n_leaf, int64_t n_head, int32_t H,
               int32_t E, int32_t C, int64_t loss_word, cudaStream_t s, bool shared = false);
int rvnn_pass(void* ctx, const float* params, const int64_t* off, float* grads, float* pool, const float* inputs,
              float* d_inputs, const uint32_t* d_blob, int64_t lv_int, int64_t lv_leaf, int64_t lv_head,
              const int32_t* lv_start, int32_t L, int64_t n_int, int64_t n_leaf, int64_t n_head, int32_t H,
              int32_t E, int32_t C, int64_t loss_word, cudaStream_t s);
int tdrnn_pass(void* ctx, const float* params, const int64_t* off, float* grads, float* pool, const float* inputs,
               float* d_inputs, const uint32_t* d_blob, int64_t lv_int, int64_t lv_leaf, int64_t lv_head,
               const int32_t* lv_start, int32_t L, int64_t n_int, int64_t n_leaf, int64_t n_head, int32_t H,
               int32_t E, int32_t C, int64_t loss_word, cudaStream_t s);
// BiLSTMwChar: the character recurrence's outputs and the rare-word lists the word tagger reads
struct CharRows {
    const uint32_t* rare;    // [T] rare index of a word position or NONE
    const uint32_t* rlist;   // [R][3] word position, character offset, length
    const float* HHc;        // [Tc][E] character h of both directions (E = 2 Hc)
};
int tagger_pass(void* ctx, const float* params, const int64_t* off, float* grads, float* pool, const float* inputs,
                float* d_inputs, const uint32_t* d_blob, int64_t tg_tok, int64_t tg_lab, int64_t tg_fpos,
                int64_t tg_bpos, const int32_t* start, int32_t maxlen, int64_t T, int32_t H, int32_t E, int32_t C,
                int32_t Mw, int32_t dirs, int64_t loss_word, cudaStream_t s, const uint32_t* chain_table = nullptr,
                int32_t chain_g = 0, const CharRows* cr = nullptr);
// BiLSTMwChar (M9): character BiLSTM (chain recurrence) -> word rows -> tagger_pass -> character backward and
// the gradients of C_emb and the character LSTMs.  off: the 17 parameter offsets in vpps.h order.
int bilstmchar_pass(void* ctx, const float* params, const int64_t* off, float* grads, float* pool,
                    const float* inputs, float* d_inputs, const uint32_t* d_blob, int64_t tg_tok, int64_t tg_lab,
                    int64_t tg_fpos, int64_t tg_bpos, const int32_t* start, int32_t maxlen, int64_t T, int32_t H,
                    int32_t E, int32_t C, int32_t Mw, int64_t loss_word, cudaStream_t s, const uint32_t* chain_table,
                    int32_t chain_g, int64_t tc_T, int64_t tc_R, int64_t tc_tok, int64_t tc_word, int64_t tc_rare,
                    int64_t tc_list, int64_t tc_chain, int32_t chain_gc, int32_t Ec);
int gru_pass(void* ctx, const float* params, const int64_t* off, float* grads, float* pool, const float* inputs,
             float* d_inputs, const uint32_t* d_blob, int64_t tg_tok, int64_t tg_lab, int64_t tg_fpos,
             const int32_t* start, int32_t maxlen, int64_t T, int32_t H, int32_t E, int32_t C, int64_t loss_word,
             cudaStream_t s, const uint32_t* chain_table = nullptr, int32_t chain_g = 0);

}  // namespace vpps
