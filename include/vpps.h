/*
 * vpps.h — C ABI of the B200-native VPPS hot path (libvpps.so).
 *
 * VPPS (Khorasani et al., MICRO'18; /root/reference/PAPER.md) trains dynamic neural nets with the
 * model's weight matrices cached in the register files of all SMs for a whole forward-backward
 * pass, driven by a per-batch instruction script generated on the host (§III).
 * The paper's user API is three calls (L191-201):
 *     vpps::handle hndl(model);               -> vpps_define_model (+ vpps_bind_buffers)
 *     float staleLoss = hndl.fb(model,cg,loss) -> vpps_build_script + vpps_fwd_bwd_sgd
 *     float latest = hndl.sync_get_latest_loss -> vpps_sync_get_latest_loss
 * and, for data parallelism across GPUs (north_star), vpps_fwd_bwd (gradients only) followed by
 * the caller's NCCL all-reduce of the gradient buffer and vpps_sgd_step.
 *
 * Conventions
 *  - Every call returns a vpps_status; no exception crosses the ABI.  On error the thread-local
 *    message is available from vpps_last_error() and no partially built object is returned.
 *  - "dev" pointers are CUDA device pointers, "host" pointers are CPU memory.
 *  - Streams are passed as void* (a cudaStream_t; NULL = legacy default stream).
 *  - A model handle is not thread-safe; use one stream per model.
 *  - Asynchronous CUDA faults surface at the next synchronising call as VPPS_E_CUDA.
 *  - The exact integer artefacts (partition table, script words, pool plan) follow SPEC_SCRIPT.md.
 */
#ifndef VPPS_H
#define VPPS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    VPPS_OK = 0,
    VPPS_E_INVALID = -1, /* bad argument (shape, null pointer, unsupported option)               */
    VPPS_E_NOFIT = -2,   /* weights do not fit the on-chip budget of any built kernel variant     */
    VPPS_E_CUDA = -3,    /* a CUDA runtime call failed (message in vpps_last_error)             */
    VPPS_E_GRAPH = -4,   /* bad graph: arity, order (children must precede parents), multiple
                            parents, token/label out of range, an empty batch (no nodes; the
                            tagger-script cells BiLSTM / GRU run it as a T = 0 pass instead)     */
    VPPS_E_STATE = -5,   /* wrong call order: buffers not bound, plan-only model, script of
                            another model                                                       */
    VPPS_E_NOMEM = -6
} vpps_status;

typedef struct vpps_model_s* vpps_model;   /* owns the partition plan, device pool, pinned staging */
typedef struct vpps_script_s* vpps_script; /* owns one batch's encoded words (host + device copy)  */

/* Cell families ("op sets").  Gate stacking inside each matrix is fixed (oracle/models.py):
 *   LSTM         (M1; Gers et al. [4]): gates (i, f, o, g)
 *   TREE_BINARY  (M4; Tai et al. [5] N=2): W_iou/U_iou rows (i, o, u)
 *   TREE_CHILDSUM(M3; Tai et al. [5] eqs. 2-8): (i, o, u)                                   */
typedef enum {
    VPPS_CELL_LSTM = 0,
    VPPS_CELL_TREE_BINARY = 1,
    VPPS_CELL_TREE_CHILDSUM = 2,
    VPPS_CELL_BILSTM_TAGGER = 3,  /* M2: forward + backward LSTM (i, f, o, g), per
                                     position m = tanh(W_mlp [h→; h←] + b_mlp), tag head z = W_tag m +
                                     b_tag; runs on the level-synchronous path (C <= 32 tags) */
    VPPS_CELL_GRU = 4,            /* M5 (the variation PAPER L21 names; DESIGN reading R-34): chains,
                                     gates (r, z, n), parameters W 3H×E, U 3H×H, W_out C×H, b_i 3H,
                                     b_h 3H, b_out C; r = σ(W_r x + b_ir + U_r h + b_hr), z likewise,
                                     n = tanh(W_n x + b_in + r ⊙ (U_n h + b_hn)), h' = (1−z) n + z h;
                                     head on labelled positions; level-synchronous path */
    VPPS_CELL_RVNN = 5,           /* M6 (DESIGN reading R-35): binary trees, untied weights
                                     W_leaf H×E, W_int H×2H, W_out C×H, b_leaf H, b_int H, b_out C;
                                     leaf h = tanh(W_leaf x + b_leaf), internal h = tanh(W_int [h_l; h_r]
                                     + b_int); level-synchronous path */
    VPPS_CELL_TDRNN = 6,          /* M7 (DESIGN reading R-36): DAGs — leaves are the input
                                     rows themselves (E = H), every inner node h = tanh(W [h_a; h_b] + b)
                                     with W H×2H, b H, and a node may feed two parents; W_out C×H, b_out C;
                                     level-synchronous path */
    VPPS_CELL_TDLSTM = 7,         /* M8 (DESIGN reading R-37): TREE_BINARY's cell and
                                     parameters on TD pyramid DAGs (a node may feed two parents, its dh and
                                     dc accumulate from both); level-synchronous path */
    VPPS_CELL_BILSTM_CHAR = 8     /* M9 BiLSTMwChar (DESIGN reading R-38): the BiLSTM tagger
                                     whose rare words (a node with a character spelling, vpps_batch.chars)
                                     take [h→ after the last character; h← after the first] of a character
                                     BiLSTM (hidden E/2 per direction, table C_emb Vc × Ec) as their input row;
                                     their table rows get no gradient, C_emb does.  Chain recurrences for the
                                     characters and the words; needs E/2 and H among the chain sizes */
} vpps_cell;

typedef struct {
    int32_t cell; /* vpps_cell                                            */
    int32_t E;    /* input (word-vector) length                           */
    int32_t H;    /* hidden length                                        */
    int32_t C;    /* classes of the softmax-NLL head          */
    int32_t mlp;  /* BiLSTM tagger MLP width M (256); ignored by the other cells */
} vpps_opset;

/* Parameter shapes, matrices first then biases (bias = {n, 1}), in exactly this order:
 *   LSTM:          W 4H×E, U 4H×H, W_out C×H, b 4H, b_out C
 *   TREE_BINARY:   W_iou 3H×E, U_iou 3H×2H, U_fl H×H, U_fr H×H, W_out C×H, b_iou 3H, b_f H, b_out C
 *   TREE_CHILDSUM: W_iou 3H×E, W_f H×E, U_iou 3H×H, U_f H×H, W_out C×H, b_iou 3H, b_f H, b_out C
 *   BILSTM_TAGGER: Wf 4H×E, Uf 4H×H, Wb 4H×E, Ub 4H×H, W_mlp M×2H, W_tag C×M, bf 4H, bb 4H, b_mlp M, b_tag C
 *   BILSTM_CHAR:   the tagger's matrices, C_emb Vc×Ec, Wcf 4Hc×Ec, Ucf 4Hc×Hc, Wcb 4Hc×Ec, Ucb 4Hc×Hc, then the
 *                  tagger's biases, bcf 4Hc, bcb 4Hc (Hc = E/2; Vc, Ec from C_emb's shape) */
typedef struct {
    int32_t rows, cols;
} vpps_shape;

/* Device-memory callbacks (PyTorch supplies device memory): the library takes its
 * activation pool, per-slot script buffers and level-path work buffers through them.  `stream` is the
 * cudaStream_t of the call that needs the memory: an allocation is used on it in stream order, and a
 * buffer is handed to free once no later work on that stream reads it (stream-ordered, like
 * cudaMallocAsync / cudaFreeAsync, so growing the pool never synchronises the device).  alloc returns
 * NULL on failure (-> VPPS_E_NOMEM).  Both NULL = cudaMallocAsync / cudaFreeAsync on `stream`.  The
 * Python binding passes torch's caching allocator. */
typedef void* (*vpps_alloc_fn)(size_t bytes, void* stream, void* ctx);
typedef void (*vpps_free_fn)(void* ptr, void* stream, void* ctx);

typedef struct {
    int32_t n_sm;        /* SMs to spread the weights over; 0 = all SMs of `device`            */
    int32_t ctas_per_sm; /* 1 (0 = auto = 1)                                                   */
    int32_t groups;      /* replica groups G (SPEC P1); 0 = 1; < 0 = automatic: the grid kernel of
                            the tree cells takes the most replicas (4, 2, 1) with a built
                            specialisation, every other path G = 1 (vpps_define_model)            */
    int32_t device;      /* CUDA device ordinal; ignored when plan_only                         */
    int32_t plan_only;   /* 1: no CUDA calls (partition + script generation only, CPU tests)   */
    int32_t cluster;     /* > 1: each replica group is one thread-block cluster of this many CTAs
                            that owns whole graphs (SPEC S5g), synchronised by the hardware
                            cluster barrier; groups = the number of co-resident clusters (or the
                            given `groups` when plan_only).  0 = grid-wide groups (SPEC S5). */
    int32_t dataflow;    /* 1 (with cluster = H / 16): the groups are ordinary co-resident CTAs of a
                            cooperative launch, one per SM (floor(n_sm / cluster) groups), and the
                            signal/wait of L165 is replaced by epoch-tagged 64-bit slots that consumers
                            poll (vpps_df); 0 = barrier synchronisation. */
    int32_t level;       /* binary cell only.  1: level-synchronous GEMM path — per level one dense
                            product of the gathered children rows with the weights (PAPER L185's
                            concatenation applied to every matrix use; weights L2-resident, plain
                            FP32 SGEMM), fused cell / head / scatter kernels, dW as one GEMM per
                            matrix.  0 = auto: chosen when no register-resident specialisation
                            exists for (H, E) (config 5: H = E = 1024); -1 = never. */
    int32_t chain;       /* chain cells on the level path (LSTM LM, BiLSTM tagger, GRU): 0 = the register-
                            resident recurrence (vpps_chain.cu) when a specialisation exists for H; -1 =
                            one recurrent product + cell launch per time step */
    vpps_alloc_fn alloc; /* device allocator for library-owned buffers (see above); NULL = default */
    vpps_free_fn free;
    void* alloc_ctx;     /* passed back to alloc / free                                         */
} vpps_options;

/* A batch of graphs in CSR form (the super-graph of L205 is built from it).
 * Node v of graph g is node graph_ptr[g] + v; its children are children[child_ptr[n] ..
 * child_ptr[n+1]) as graph-local indices that must precede v (children-first order). */
typedef struct {
    int32_t n_graphs;
    const int32_t* graph_ptr; /* host [n_graphs+1]                                   */
    const int32_t* child_ptr; /* host [n_nodes+1]                                    */
    const int32_t* children;  /* host [child_ptr[n_nodes]] graph-local indices       */
    const int32_t* token;     /* host [n_nodes] input-table row or -1                */
    const int32_t* label;     /* host [n_nodes] class of a loss head on this node, or -1 */
    const int32_t* char_ptr;  /* host [n_nodes+1] or NULL: node v's spelling is chars[char_ptr[v] ..
                                 char_ptr[v+1]) (BILSTM_CHAR only; an empty spelling = a frequent word) */
    const int32_t* chars;     /* host character ids in [0, Vc)                      */
} vpps_batch;

typedef struct {
    int64_t n_words;      /* script words (header + streams + barrier targets)        */
    int64_t pool_words;   /* activation pool size in 4-byte words (SPEC §S7)          */
    int64_t zero_words;   /* leading pool words cleared before every pass            */
    int64_t loss_word;    /* pool word holding the summed batch loss                  */
    int32_t n_barriers;   /* 2L+1                                                      */
    int32_t n_levels;     /* L+1                                                       */
    int64_t n_nodes;      /* super-graph nodes (cells + heads)                          */
    int64_t n_heads;
    double flops;         /* algorithmic FLOPs of the pass (2/MAC; fwd, dW, dX/dh)     */
    double act_bytes;     /* algorithmic activation bytes read+written by the pass     */
    int64_t blob_words;   /* words copied host->device per pass: the script words plus the device-side
                             node lists and dataflow program (the one H2D copy of L169)  */
    double kernel_flops;  /* algorithmic FLOPs of the replica-group kernel of the binary cluster /
                             dataflow paths (internal-cell matvecs and transposed products, 32 H^2
                             per cell, and the loss heads); the rest of `flops` runs in the GEMMs */
} vpps_script_info;

/* ---- model (vpps::handle hndl(model)) -------------------------------------- */

/* Validates the shapes against the op set, builds the partition plan (SPEC §P1) and selects the
 * kernel specialisation (templated on cell, H, E and units per CTA; Fig.5). */
vpps_status vpps_define_model(const vpps_shape* params, int32_t n_params, const vpps_opset* ops,
                              const vpps_options* opt, vpps_model* out);

/* Flat float layout of the parameters: total floats and the offset of each parameter (16-byte
 * aligned).  params_flat and grads_flat below use this layout (row-major, PAPER fn3 L98). */
vpps_status vpps_layout(vpps_model m, int64_t* n_floats, int64_t* offsets /* [n_params] */);

/* Binds caller-owned device buffers (e.g. torch tensors): the DRAM master copy of the
 * parameters and the gradient buffer (same layout).  Not copied. */
vpps_status vpps_bind_buffers(vpps_model m, float* params_flat /*dev*/, float* grads_flat /*dev*/);

/* Partition table (SPEC P1.6): n rows of 8 int32 (matrix,row,cols,group,cta,slot,storage,
 * grad_storage).  Pointer valid until the model is destroyed. */
vpps_status vpps_partition_table(vpps_model m, const int32_t** rows8, int64_t* n_rows);

/* Plan summary: n_cta, CTAs per group, active CTAs per group, units per CTA (UMAX). */
vpps_status vpps_plan_info(vpps_model m, int32_t* n_cta, int32_t* n_g, int32_t* n_act, int32_t* umax);

/* Paper-literal dealer (SPEC P0; Fig.4, Eq.(1), fn6): writes rows of 6 int32
 * (matrix,row,cta,partition,warp,is_grad) into out6 (host, may be NULL to query the size). */
vpps_status vpps_paper_deal(const vpps_shape* mats, int32_t n_mats, int32_t n_cta, int32_t tb,
                            int32_t rpw, int32_t pack_rows, int32_t grads, int32_t* out6,
                            int64_t* n_rows, int64_t* n_slots);
/* P0.7: 2 if everything fits in registers at two CTAs per SM, else 1. */
int32_t vpps_paper_choose_cps(const vpps_shape* mats, int32_t n_mats, int32_t n_sm, int32_t tb,
                              int32_t rpw, int32_t pack_rows);

/* ---- script (PAPER §III-B1) -------------------------------------------------- */

/* Lowers a batch to per-group instruction streams (level sort L139, forward/backward traversal
 * L141/L167, signal/wait L165, pool plan L159) and stages the words in pinned host memory.
 * The batch arrays are deep-copied; the caller may free them on return. */
vpps_status vpps_build_script(vpps_model m, const vpps_batch* batch, vpps_script* out);
/* The SPEC words (SPEC_SCRIPT.md §E).  A dataflow model's scripts leave them out of the device blob (its
 * kernels never read them); they are built here on first request (same batch, same result). */
vpps_status vpps_script_words(vpps_script s, const uint32_t** words /*host*/, int64_t* n_words);
/* The whole device upload blob (host copy; SPEC_SCRIPT.md §D/§L): [words ‖] the device lowerings.
 * *lists_off = blob offset of the device lowering (0 when the words are left out), *df_off = offset of
 * the dataflow program or -1.  Pointer valid until the script is destroyed. */
vpps_status vpps_script_blob(vpps_script s, const uint32_t** blob /*host*/, int64_t* n_words,
                             int64_t* lists_off, int64_t* df_off);
vpps_status vpps_script_info_get(vpps_script s, vpps_script_info* info);
/* Asynchronous H2D copy of the script (one copy).  vpps_fwd_bwd* upload a script
 * automatically on first use; call this to move the copy out of the timed kernel region. */
vpps_status vpps_upload_script(vpps_script s, void* stream);

/* ---- training step --------------------------------------------------------------------- */

/* One persistent kernel launch: prologue (weights DRAM->registers), script
 * interpretation (L171-177), epilogue.  Writes the gradient of the summed loss (L205) into
 * grads_flat and, if d_inputs != NULL, the gradient w.r.t. the input table into d_inputs
 * (overwritten).  inputs: dev [n_input_rows × E] row-major (token t = row t). Asynchronous. */
vpps_status vpps_fwd_bwd(vpps_model m, vpps_script s, const float* inputs, int64_t n_input_rows,
                         float* d_inputs, void* stream);

/* params ← params − lr·(grads + weight_decay·params) over the whole flat buffer (PAPER L129,
 * L197: weight decay queried from the model).  Use after an all-reduce of grads_flat. */
vpps_status vpps_sgd_step(vpps_model m, float lr, float weight_decay, void* stream);

/* The paper's single-kernel mode (L25, L84): forward, backward and the SGD update in one launch;
 * grads_flat is not written. */
vpps_status vpps_fwd_bwd_sgd(vpps_model m, vpps_script s, const float* inputs, int64_t n_input_rows,
                             float* d_inputs, float lr, float weight_decay, void* stream);

/* Stale loss: the summed loss of the previous completed pass (0 before any), after
 * waiting for that pass only.  Latest loss (L201): waits for the most recent pass. */
vpps_status vpps_get_stale_loss(vpps_model m, float* loss);
vpps_status vpps_sync_get_latest_loss(vpps_model m, float* loss);

/* Measurement hook: when set (cudaEvent_t handles, or NULL to clear), every later launch records
 * ev_before immediately before and ev_after immediately after the persistent kernel on the
 * launching stream, so the kernel's own duration can be timed without the pool memsets. */
vpps_status vpps_set_timing_events(vpps_model m, void* ev_before, void* ev_after);

/* Measurement hook for the replica-group kernel alone (cluster / dataflow paths): ev_before and ev_after
 * are recorded immediately around vpps_cl / vpps_df only.  The records sit between programmatically
 * dependent launches, so while set the neighbouring GEMMs no longer overlap that kernel: use it for a
 * separate timing pass.  NULL clears. */
vpps_status vpps_set_kernel_events(vpps_model m, void* ev_before, void* ev_after);

/* In-kernel phase trace (measurement only): when buf != NULL (dev, >= n_cta*stride uint64), every
 * later launch writes per CTA, from %globaltimer (ns): [0] start of interpretation, [1] end, and for
 * barrier b: [2+3b] signal, [3+3b] wait begin, [4+3b] wait end.  stride >= 2 + 3*(n_barriers+1). */
vpps_status vpps_set_profile_buffer(vpps_model m, uint64_t* buf, int64_t stride);

/* Measurement hook (dataflow path): when buf != NULL (dev, >= 5 x gradient-GEMM items uint64), every
 * later pass writes per item of the gradient GEMM (group, item, start ns, end ns, SM id). */
vpps_status vpps_set_gemm_trace(vpps_model m, uint64_t* buf);

/* Device pointer of the model's activation pool (SPEC §S7 layout of the last script run). */
vpps_status vpps_pool_ptr(vpps_model m, float** pool, int64_t* pool_words);

/* The level paths' dense FP32 product (PAPER L185's concatenated operands; hand-written FFMA2 tiles,
 * csrc/kernels/vpps_gemm.cu), exposed for testing:  C = op(A) op(B) + beta C, row-major dev pointers,
 * op(A) = A (M x K, leading dimension lda) or, with ta, the transpose of A stored K x M; op(B) = B (K x N)
 * or, with tb, the transpose of B stored N x K.  beta must be 0 or 1.  Asynchronous on `stream`; returns
 * a vpps_status: VPPS_E_INVALID for bad arguments, VPPS_E_CUDA for a failed launch. */
int32_t vpps_gemm_f32(void* stream, int32_t ta, int32_t tb, int32_t M, int32_t N, int32_t K, const float* A,
                      int32_t lda, const float* B, int32_t ldb, float* C, int32_t ldc, float beta);

void vpps_destroy_script(vpps_script s);
void vpps_destroy_model(vpps_model m);
const char* vpps_last_error(void);
/* Kernel specialisations compiled into this library: writes up to cap entries of
 * (cell, H, E, umax) into out4 and returns the count. */
int32_t vpps_variants(int32_t* out4, int32_t cap);

#ifdef __cplusplus
}
#endif
#endif /* VPPS_H */
