// C ABI of libvpps (include/vpps.h): argument checking, object lifetime, the one H2D script copy,
// the cooperative launch of the persistent kernel and loss bookkeeping.  No torch types here.
#include <cuda_runtime.h>
#include <algorithm>
#include <climits>
#include <cstring>
#include <memory>
#include <new>
#include <string>
#include <vector>

#include "../../include/vpps.h"
#include "host/host.h"
#include "kernels/vpps_kernel.cuh"

using namespace vpps;

namespace {
thread_local std::string g_err;

vpps_status fail(vpps_status st, const std::string& msg) {
    g_err = msg;
    return st;
}
vpps_status cuda_fail(cudaError_t e, const char* what) {
    g_err = std::string(what) + ": " + cudaGetErrorString(e);
    return VPPS_E_CUDA;
}
#define CK(call)                                               \
    do {                                                       \
        cudaError_t _e = (call);                               \
        if (_e != cudaSuccess) return cuda_fail(_e, #call);    \
    } while (0)

std::vector<Shape> expected_shapes(int32_t cell, int32_t H, int32_t E, int32_t C, int32_t M = 0, int32_t Vc = 0,
                                   int32_t Ec = 0) {
    const int32_t Hc = E / 2;
    switch (cell) {
        case CELL_BILSTM_CHAR:
            return {{4 * H, E}, {4 * H, H}, {4 * H, E}, {4 * H, H}, {M, 2 * H}, {C, M}, {Vc, Ec}, {4 * Hc, Ec},
                    {4 * Hc, Hc}, {4 * Hc, Ec}, {4 * Hc, Hc}, {4 * H, 1}, {4 * H, 1}, {M, 1}, {C, 1}, {4 * Hc, 1},
                    {4 * Hc, 1}};
        case CELL_BILSTM:
            return {{4 * H, E}, {4 * H, H}, {4 * H, E}, {4 * H, H}, {M, 2 * H}, {C, M},
                    {4 * H, 1}, {4 * H, 1}, {M, 1}, {C, 1}};
        case CELL_LSTM: return {{4 * H, E}, {4 * H, H}, {C, H}, {4 * H, 1}, {C, 1}};
        case CELL_GRU: return {{3 * H, E}, {3 * H, H}, {C, H}, {3 * H, 1}, {3 * H, 1}, {C, 1}};
        case CELL_RVNN: return {{H, E}, {H, 2 * H}, {C, H}, {H, 1}, {H, 1}, {C, 1}};
        case CELL_TDRNN: return {{H, 2 * H}, {C, H}, {H, 1}, {C, 1}};
        case CELL_BINARY:
        case CELL_TDLSTM: return {{3 * H, E}, {3 * H, 2 * H}, {H, H}, {H, H}, {C, H}, {3 * H, 1}, {H, 1}, {C, 1}};
        case CELL_CHILDSUM: return {{3 * H, E}, {H, E}, {3 * H, H}, {H, H}, {C, H}, {3 * H, 1}, {H, 1}, {C, 1}};
    }
    return {};
}
}  // namespace

struct vpps_model_s {
    Plan plan;
    DevAlloc alloc;                     // device memory of library-owned buffers (vpps_options callbacks)
    std::vector<Shape> shapes;
    std::vector<int64_t> offsets;
    int64_t n_floats = 0;
    bool plan_only = true;
    int device = 0;
    int32_t sms = 148;                  // SM count of the device (persistent GEMM grids)
    const Variant* var = nullptr;
    size_t smem = 0;
    float* params = nullptr;
    float* grads = nullptr;
    float* pool = nullptr;
    int64_t pool_cap = 0, last_pool_words = 0;
    float* h_loss = nullptr;            // pinned [2] (mapped on the cluster / dataflow paths)
    float* d_loss_map = nullptr;        // device view of h_loss (kernel writes the loss directly)
    cudaEvent_t ev[2] = {nullptr, nullptr};
    int64_t passes = 0;
    cudaEvent_t t_before = nullptr, t_after = nullptr;
    cudaEvent_t k_before = nullptr, k_after = nullptr;   // around the replica-group kernel only
    uint64_t* gemm_trace = nullptr;                      // measurement: gradient GEMM item stamps
    uint64_t* prof = nullptr;
    int64_t prof_stride = 0;
    int32_t cluster = 0;                // > 1: cluster-replica path (vpps_cluster.cu)
    int32_t* done = nullptr;            // per-group completion counters [kMaxGroups] + GEMM claim counters [kMaxGroups]
    bool dataflow = false;              // groups of co-resident CTAs synchronised by tagged slots (vpps_df)
    uint32_t* d_epoch = nullptr;        // dataflow pass counter on the device (slot tags), advanced per pass
    static constexpr int kMaxGroups = 16;
    void* level = nullptr;              // level-synchronous path context (second stream, work buffers)
    // Pre-allocated staging ring for per-batch scripts: a pinned host buffer and a
    // device buffer per slot; a slot is reused once the kernel that last read it has finished.
    struct Slot {
        uint32_t* h = nullptr;
        uint32_t* d = nullptr;
        size_t cap = 0;
        cudaEvent_t done = nullptr;
        bool used = false;
    };
    static constexpr int kSlots = 3;
    Slot ring[kSlots];
    int next_slot = 0;
};

struct vpps_script_s {
    vpps_model model = nullptr;
    Script s;
    // dataflow models build the SPEC words on request only (Plan::skip_words): the batch is kept for that
    bool words_pending = false;
    std::vector<int32_t> b_gp, b_cp, b_ch, b_tok, b_lab;
    uint32_t* d_words = nullptr;   // dedicated device copy after vpps_upload_script (resident script)
    bool uploaded = false;
};

extern "C" {

const char* vpps_last_error(void) { return g_err.c_str(); }

int32_t vpps_variants(int32_t* out4, int32_t cap) {
    int32_t n = 0;
    const Variant* v = variants(&n);
    for (int32_t i = 0; i < n && i < cap && out4; ++i) {
        out4[4 * i] = v[i].cell; out4[4 * i + 1] = v[i].H; out4[4 * i + 2] = v[i].E; out4[4 * i + 3] = v[i].umax;
    }
    return n;
}

vpps_status vpps_define_model(const vpps_shape* params, int32_t n_params, const vpps_opset* ops,
                              const vpps_options* opt, vpps_model* out) {
    if (!params || !ops || !out) return fail(VPPS_E_INVALID, "null argument");
    *out = nullptr;
    vpps_options o{};
    if (opt) o = *opt;
    if (o.groups < 0) {
        // automatic replica groups (SPEC P1 from the register budget): on the grid kernel of the tree cells
        // (child-sum, binary without clusters / forced level path) the most replicas that fit a built
        // specialisation — G = 4, 2, 1 — since more replicas of the weights process more graphs at once
        // (config 2: 1.15 / 0.67 / 0.43 ms for G = 1 / 2 / 4; TGT on the grid kernel 0.51 / 0.36 / 0.31 ms,
        // profiles/r2_grid_groups_sweep.jsonl); every other path keeps G = 1
        vpps_options o2 = o;
        const bool grid_tree = (ops->cell == CELL_CHILDSUM || ops->cell == CELL_BINARY) && o.cluster <= 1 &&
                               !o.dataflow && o.level <= 0;
        if (grid_tree) {
            for (int32_t g : {4, 2}) {
                o2.groups = g;
                if (vpps_define_model(params, n_params, ops, &o2, out) == VPPS_OK) return VPPS_OK;
            }
        }
        o2.groups = 1;
        return vpps_define_model(params, n_params, ops, &o2, out);
    }
    const int32_t cell = ops->cell, H = ops->H, E = ops->E, C = ops->C, Mw = ops->mlp;
    if (cell < 0 || cell > 8 || H <= 0 || E <= 0 || C <= 0) return fail(VPPS_E_INVALID, "bad op set");
    if (cell == CELL_TDRNN && E != H) return fail(VPPS_E_INVALID, "TD-RNN: the leaves are the input rows (E == H)");
    if ((cell == CELL_BILSTM || cell == CELL_BILSTM_CHAR) && Mw <= 0)
        return fail(VPPS_E_INVALID, "BiLSTM tagger needs mlp > 0");
    // BiLSTMwChar: the character table's shape (parameter 6, Vc x Ec) sets Vc and Ec; E must be even
    const int32_t Vc = cell == CELL_BILSTM_CHAR && n_params > 6 ? params[6].rows : 0;
    const int32_t Ec = cell == CELL_BILSTM_CHAR && n_params > 6 ? params[6].cols : 0;
    if (cell == CELL_BILSTM_CHAR && (E % 2 || Vc <= 0 || Ec <= 0 || Ec % 4))
        return fail(VPPS_E_INVALID, "BiLSTMwChar: E even, C_emb Vc x Ec with Ec a multiple of 4");
    std::vector<Shape> want = expected_shapes(cell, H, E, C, Mw, Vc, Ec);
    if ((int32_t)want.size() != n_params) return fail(VPPS_E_INVALID, "wrong number of parameters for the op set");
    for (int32_t i = 0; i < n_params; ++i)
        if (params[i].rows != want[i].rows || params[i].cols != want[i].cols)
            return fail(VPPS_E_INVALID, "parameter " + std::to_string(i) + " has the wrong shape for the op set");
    if (o.groups == 0) o.groups = 1;
    if (o.ctas_per_sm == 0) o.ctas_per_sm = 1;
    if (o.ctas_per_sm != 1) return fail(VPPS_E_INVALID, "ctas_per_sm must be 1 in v1");

    std::unique_ptr<vpps_model_s> m(new (std::nothrow) vpps_model_s);
    if (!m) return fail(VPPS_E_NOMEM, "out of host memory");
    m->plan_only = o.plan_only != 0;
    if ((o.alloc == nullptr) != (o.free == nullptr)) return fail(VPPS_E_INVALID, "alloc and free callbacks go together");
    m->alloc.alloc_fn = o.alloc;
    m->alloc.free_fn = o.free;
    m->alloc.ctx = o.alloc_ctx;
    m->shapes = want;
    int64_t cur = 0;
    for (const Shape& s : want) {
        m->offsets.push_back(cur);
        cur += ((int64_t)s.rows * s.cols + 3) / 4 * 4;
    }
    m->n_floats = cur;
    int32_t n_sm = o.n_sm;
    if (cell == CELL_BILSTM || cell == CELL_BILSTM_CHAR || cell == CELL_GRU || cell == CELL_RVNN || cell == CELL_TDRNN ||
        cell == CELL_TDLSTM ||
        (cell == CELL_LSTM &&
         (o.level > 0 ||
          (o.level == 0 && (C > 32 || (o.chain >= 0 && o.groups <= 1 && H >= 128 && chain_group_ctas(H) > 0)))))) {
        // (an LSTM at H >= 128 takes the chain recurrence + dense products by default — 3.6x the grid kernel
        //  at config 3, H = 256; at config 1's H = 32 the one-kernel grid path is faster, 0.054 vs 0.093 ms;
        //  level = -1 / 1 force either)
        // M2 and M5 (GRU) run on the level-synchronous path only (vpps_level.cu), and so does an LSTM LM
        // whose vocabulary head exceeds one CTA's shared memory (config 3 at V = 1000): no partition plan
        if (o.cluster > 1 || o.dataflow || o.level < 0) return fail(VPPS_E_INVALID, "this op set runs on the level path only");
        if (H % 4 || E % 4) return fail(VPPS_E_INVALID, "H and E must be multiples of 4");
        if (cell == CELL_LSTM) {
            // the partition plan (SPEC P1) stays defined for the op set (a bit-exact artifact) even though
            // the level path does not place weights by it
            std::string perr;
            if (!unit_plan(cell, H, E, C, n_sm ? n_sm : 148, o.ctas_per_sm, o.groups, &m->plan, &perr))
                return fail(perr.rfind("NOFIT", 0) == 0 ? VPPS_E_NOFIT : VPPS_E_INVALID, perr);
        } else {
            m->plan.cell = cell; m->plan.H = H; m->plan.E = E; m->plan.C = C;
            m->plan.n_cta = m->plan.n_g = m->plan.n_act = m->plan.umax = m->plan.G = 1;
        }
        m->plan.mlp = cell == CELL_BILSTM || cell == CELL_BILSTM_CHAR ? Mw : 0;
        m->plan.vc = Vc;
        m->plan.ec = Ec;
        m->plan.level = true;
        int32_t sms = 148;
        if (!m->plan_only) {
            m->device = o.device;
            CK(cudaSetDevice(o.device));
            cudaDeviceProp prop;
            CK(cudaGetDeviceProperties(&prop, o.device));
            if (prop.major != 10) return fail(VPPS_E_INVALID, "libvpps is built for sm_100a (B200) only");
            sms = prop.multiProcessorCount;
        }
        // LSTM chains: the recurrence runs register-resident in groups of co-resident CTAs (vpps_chain.cu)
        // when a specialisation exists for H; VPPS_CHAIN=0 (measurement) keeps the per-step products
        static const bool chain_env = !(getenv("VPPS_CHAIN") && atoi(getenv("VPPS_CHAIN")) == 0);
        if ((cell == CELL_BILSTM || cell == CELL_BILSTM_CHAR || cell == CELL_LSTM || cell == CELL_GRU) && chain_env &&
            o.chain >= 0) {
            const int32_t ncl = chain_group_ctas(H), dirs = cell == CELL_BILSTM || cell == CELL_BILSTM_CHAR ? 2 : 1;
            m->plan.chain_g = ncl > 0 ? (sms / ncl) / dirs : 0;
        }
        if (cell == CELL_BILSTM_CHAR) {
            // the character BiLSTM runs only on the chain recurrence (H_c = E / 2 must be a built size)
            const int32_t ncl = chain_group_ctas(E / 2);
            if (ncl <= 0) return fail(VPPS_E_NOFIT, "BiLSTMwChar: no chain specialisation for H_c = E / 2");
            m->plan.chain_gc = (sms / ncl) / 2;
        }
        if (!m->plan_only) {
            m->level = level_ctx_create(&m->alloc);
            if (!m->level) return fail(VPPS_E_CUDA, "level-path context initialisation failed");
            CK(cudaMallocHost(&m->h_loss, 2 * sizeof(float)));
            m->h_loss[0] = m->h_loss[1] = 0.f;
            CK(cudaEventCreateWithFlags(&m->ev[0], cudaEventDisableTiming));
            CK(cudaEventCreateWithFlags(&m->ev[1], cudaEventDisableTiming));
        }
        *out = m.release();
        return VPPS_OK;
    }
    m->cluster = o.cluster > 1 ? o.cluster : 0;
    m->dataflow = m->cluster && o.dataflow;
    if (!m->plan_only) {
        m->device = o.device;
        CK(cudaSetDevice(o.device));
        cudaDeviceProp prop;
        CK(cudaGetDeviceProperties(&prop, o.device));
        if (prop.major != 10) return fail(VPPS_E_INVALID, "libvpps is built for sm_100a (B200) only");
        if (n_sm == 0) n_sm = prop.multiProcessorCount;
        if (n_sm > prop.multiProcessorCount) return fail(VPPS_E_INVALID, "n_sm exceeds the device's SM count");
        m->sms = prop.multiProcessorCount;
    } else if (n_sm == 0) {
        n_sm = m->cluster ? m->cluster * o.groups : 148;
    }
    if (m->dataflow && !m->plan_only) {
        // dataflow groups (SPEC S5g): floor(n_sm / cluster) groups of co-resident CTAs (cooperative launch)
        int32_t nv = 0;
        const Variant* v = df_variants(&nv);
        for (int32_t i = 0; i < nv; ++i)
            if (v[i].cell == cell && v[i].H == H && v[i].E == E && v[i].umax == m->cluster) m->var = &v[i];
        if (!m->var) return fail(VPPS_E_NOFIT, "no dataflow specialisation for this op set and group size");
        if (C > 32) return fail(VPPS_E_NOFIT, "single-CTA loss head supports C <= 32 classes in v1");
        m->smem = m->var->smem_bytes(C);
        CK(cudaFuncSetAttribute(m->var->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)m->smem));
        int per_sm = 0;
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, m->var->fn, df_block(m->var->fn), m->smem));
        if (per_sm < 1) return fail(VPPS_E_NOFIT, "dataflow kernel does not fit on an SM");
        o.groups = std::min(n_sm / m->cluster, vpps_model_s::kMaxGroups);
        if (o.groups < 1) return fail(VPPS_E_NOFIT, "fewer SMs than one group");
        n_sm = o.groups * m->cluster;
    } else if (m->cluster && !m->plan_only) {
        // cluster replicas (SPEC S5g): one group per co-resident cluster of `cluster` CTAs
        int32_t nv = 0;
        const Variant* v = cluster_variants(&nv);
        for (int32_t i = 0; i < nv; ++i)
            if (v[i].cell == cell && v[i].H == H && v[i].E == E && v[i].umax == m->cluster) m->var = &v[i];
        if (!m->var) return fail(VPPS_E_NOFIT, "no cluster specialisation for this op set and cluster size");
        if (C > 32) return fail(VPPS_E_NOFIT, "single-CTA loss head supports C <= 32 classes in v1");
        m->smem = m->var->smem_bytes(C);
        CK(cudaFuncSetAttribute(m->var->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)m->smem));
        CK(cudaFuncSetAttribute(m->var->fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
        cudaLaunchConfig_t cfg = {};
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeClusterDimension;
        attr[0].val.clusterDim.x = m->cluster;
        attr[0].val.clusterDim.y = 1;
        attr[0].val.clusterDim.z = 1;
        cfg.gridDim = dim3(m->cluster);
        cfg.blockDim = dim3(256);
        cfg.dynamicSmemBytes = m->smem;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        int ncl = 0;
        CK(cudaOccupancyMaxActiveClusters(&ncl, m->var->fn, &cfg));
        ncl = std::min(ncl, n_sm / m->cluster);
        if (ncl < 1) return fail(VPPS_E_NOFIT, "no cluster of this size can be resident");
        o.groups = ncl;
        n_sm = ncl * m->cluster;
    }
    std::string err;
    if (!unit_plan(cell, H, E, C, n_sm, o.ctas_per_sm, o.groups, &m->plan, &err))
        return fail(err.rfind("NOFIT", 0) == 0 ? VPPS_E_NOFIT : VPPS_E_INVALID, err);
    m->plan.by_graph = m->cluster != 0;
    m->plan.skip_words = m->dataflow;   // vpps_df reads only the device lowering (SPEC §D)
    if (m->cluster && m->plan.n_g != m->cluster) return fail(VPPS_E_INVALID, "groups x cluster must equal n_sm");
    if (m->cluster && !m->plan_only) {
        if (m->plan.G > vpps_model_s::kMaxGroups) return fail(VPPS_E_NOFIT, "more than 16 cluster replicas");
        CK(setup_leaf_attrs());        // per device (this model's), after cudaSetDevice above
        CK(setup_dw_gemm_attrs());
        CK(cudaMalloc(&m->done, 4 * vpps_model_s::kMaxGroups * sizeof(int32_t)));   // done, claim, fin/tail
        CK(cudaMemset(m->done, 0, 4 * vpps_model_s::kMaxGroups * sizeof(int32_t)));
        CK(cudaMalloc(&m->d_epoch, sizeof(uint32_t)));
        CK(cudaMemset(m->d_epoch, 0, sizeof(uint32_t)));
        CK(cudaHostAlloc(&m->h_loss, 2 * sizeof(float), cudaHostAllocMapped));
        CK(cudaHostGetDevicePointer(reinterpret_cast<void**>(&m->d_loss_map), m->h_loss, 0));
        m->h_loss[0] = m->h_loss[1] = 0.f;
        CK(cudaEventCreateWithFlags(&m->ev[0], cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&m->ev[1], cudaEventDisableTiming));
    } else if (!m->plan_only) {
        if (H % 4 || E % 4) return fail(VPPS_E_INVALID, "H and E must be multiples of 4");
        int32_t nv = 0;
        const Variant* v = variants(&nv);
        for (int32_t i = 0; i < nv; ++i)
            if (v[i].cell == cell && v[i].H == H && v[i].E == E && v[i].umax == m->plan.umax) m->var = &v[i];
        const bool want_level = cell == CELL_BINARY && (o.level > 0 || (o.level == 0 && !m->var));
        if (o.level > 0 && cell != CELL_BINARY) return fail(VPPS_E_INVALID, "the level path is built for the binary cell");
        if (want_level) {
            // level-synchronous GEMM path (vpps_level.cu): no register-resident specialisation needed
            m->var = nullptr;
            m->plan.level = true;
            m->level = level_ctx_create(&m->alloc);
            if (!m->level) return fail(VPPS_E_CUDA, "level-path context initialisation failed");
            CK(cudaMallocHost(&m->h_loss, 2 * sizeof(float)));
            m->h_loss[0] = m->h_loss[1] = 0.f;
            CK(cudaEventCreateWithFlags(&m->ev[0], cudaEventDisableTiming));
            CK(cudaEventCreateWithFlags(&m->ev[1], cudaEventDisableTiming));
            *out = m.release();
            return VPPS_OK;
        }
        if (!m->var)
            return fail(VPPS_E_NOFIT, "no kernel specialisation for cell " + std::to_string(cell) + " H=" +
                                          std::to_string(H) + " E=" + std::to_string(E) +
                                          " units/CTA=" + std::to_string(m->plan.umax));
        if (C > 32) return fail(VPPS_E_NOFIT, "single-CTA loss head supports C <= 32 classes in v1");
        m->smem = m->var->smem_bytes(C);
        if (m->smem > 227 * 1024) return fail(VPPS_E_NOFIT, "head does not fit in shared memory");
        CK(cudaFuncSetAttribute(m->var->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)m->smem));
        int blocks = 0;
        CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks, m->var->fn, 256, m->smem));
        if (blocks < 1) return fail(VPPS_E_NOFIT, "kernel cannot be resident (registers/shared memory)");
        CK(cudaMallocHost(&m->h_loss, 2 * sizeof(float)));
        m->h_loss[0] = m->h_loss[1] = 0.f;
        CK(cudaEventCreateWithFlags(&m->ev[0], cudaEventDisableTiming));
        CK(cudaEventCreateWithFlags(&m->ev[1], cudaEventDisableTiming));
    }
    *out = m.release();
    return VPPS_OK;
}

vpps_status vpps_layout(vpps_model m, int64_t* n_floats, int64_t* offsets) {
    if (!m) return fail(VPPS_E_INVALID, "null model");
    if (n_floats) *n_floats = m->n_floats;
    if (offsets) std::memcpy(offsets, m->offsets.data(), m->offsets.size() * sizeof(int64_t));
    return VPPS_OK;
}

vpps_status vpps_bind_buffers(vpps_model m, float* params_flat, float* grads_flat) {
    if (!m || !params_flat || !grads_flat) return fail(VPPS_E_INVALID, "null argument");
    if (m->plan_only) return fail(VPPS_E_STATE, "plan-only model");
    if (((uintptr_t)params_flat | (uintptr_t)grads_flat) & 15) return fail(VPPS_E_INVALID, "buffers must be 16-byte aligned");
    m->params = params_flat;
    m->grads = grads_flat;
    return VPPS_OK;
}

vpps_status vpps_partition_table(vpps_model m, const int32_t** rows8, int64_t* n_rows) {
    if (!m || !rows8 || !n_rows) return fail(VPPS_E_INVALID, "null argument");
    *rows8 = m->plan.table.data();
    *n_rows = (int64_t)m->plan.table.size() / 8;
    return VPPS_OK;
}

vpps_status vpps_plan_info(vpps_model m, int32_t* n_cta, int32_t* n_g, int32_t* n_act, int32_t* umax) {
    if (!m) return fail(VPPS_E_INVALID, "null model");
    if (n_cta) *n_cta = m->plan.n_cta;
    if (n_g) *n_g = m->plan.n_g;
    if (n_act) *n_act = m->plan.n_act;
    if (umax) *umax = m->plan.umax;
    return VPPS_OK;
}

vpps_status vpps_paper_deal(const vpps_shape* mats, int32_t n_mats, int32_t n_cta, int32_t tb, int32_t rpw,
                            int32_t pack_rows, int32_t grads, int32_t* out6, int64_t* n_rows, int64_t* n_slots) {
    if (!mats || n_mats <= 0 || n_cta <= 0 || tb <= 0 || tb % 32 || rpw <= 0 || !n_rows || !n_slots)
        return fail(VPPS_E_INVALID, "bad argument");
    std::vector<Shape> v(n_mats);
    for (int32_t i = 0; i < n_mats; ++i) v[i] = {mats[i].rows, mats[i].cols};
    std::vector<DealRow> rows;
    paper_deal(v, n_cta, tb, rpw, pack_rows != 0, grads != 0, &rows, n_slots);
    *n_rows = (int64_t)rows.size();
    if (out6)
        for (size_t i = 0; i < rows.size(); ++i) {
            const DealRow& r = rows[i];
            const int32_t x[6] = {r.matrix, r.row, r.cta, r.partition, r.warp, r.is_grad};
            std::memcpy(out6 + 6 * i, x, sizeof(x));
        }
    return VPPS_OK;
}

int32_t vpps_paper_choose_cps(const vpps_shape* mats, int32_t n_mats, int32_t n_sm, int32_t tb, int32_t rpw,
                              int32_t pack_rows) {
    std::vector<Shape> v(n_mats);
    for (int32_t i = 0; i < n_mats; ++i) v[i] = {mats[i].rows, mats[i].cols};
    return paper_choose_cps(v, n_sm, tb, rpw, pack_rows != 0);
}

vpps_status vpps_build_script(vpps_model m, const vpps_batch* batch, vpps_script* out) {
    if (!m || !batch || !out) return fail(VPPS_E_INVALID, "null argument");
    *out = nullptr;
    std::unique_ptr<vpps_script_s> s(new (std::nothrow) vpps_script_s);
    if (!s) return fail(VPPS_E_NOMEM, "out of host memory");
    s->model = m;
    BatchIn b{batch->n_graphs, batch->graph_ptr, batch->child_ptr, batch->children, batch->token, batch->label,
              batch->char_ptr, batch->chars};
    std::string err;
    // the input table's row count is not known here; token range is re-checked against it at run time
    const bool chains = m->plan.level && (m->plan.cell == CELL_BILSTM || m->plan.cell == CELL_BILSTM_CHAR ||
                                          m->plan.cell == CELL_LSTM ||
                                          m->plan.cell == CELL_GRU);
    int rc = 0;
    if (chains && m->plan.cell == CELL_LSTM) {
        // LSTM LM on the level path: the SPEC script (words, pool plan: a bit-exact artifact of the op set)
        // plus the chain lists of the level path appended to the upload blob
        Plan spec = m->plan;
        spec.level = false;
        rc = build_script(spec, b, INT64_MAX, &s->s, &err);
        Script t;
        if (rc == 0) rc = build_tagger_script(m->plan, b, INT64_MAX, &t, &err);
        if (rc == 0) {
            const int64_t shift = (int64_t)s->s.blob.size();
            s->s.blob.insert(s->s.blob.end(), t.blob.begin(), t.blob.end());
            s->s.tg_T = t.tg_T;
            s->s.tg_tok = t.tg_tok + shift;
            s->s.tg_lab = t.tg_lab + shift;
            s->s.tg_fpos = t.tg_fpos + shift;
            s->s.tg_bpos = t.tg_bpos + shift;
            s->s.tg_start = t.tg_start;
            s->s.tg_chain = t.tg_chain >= 0 ? t.tg_chain + shift : -1;
        }
    } else {
        rc = chains ? build_tagger_script(m->plan, b, INT64_MAX, &s->s, &err)
                    : build_script(m->plan, b, INT64_MAX, &s->s, &err);
        if (rc == 0 && !chains && m->plan.skip_words && b.n_graphs > 0) {
            // the SPEC words are built on request (vpps_script_words): keep a copy of the batch
            const int32_t nn = b.graph_ptr[b.n_graphs];
            s->b_gp.assign(b.graph_ptr, b.graph_ptr + b.n_graphs + 1);
            s->b_cp.assign(b.child_ptr, b.child_ptr + nn + 1);
            s->b_ch.assign(b.children, b.children + b.child_ptr[nn]);
            s->b_tok.assign(b.token, b.token + nn);
            s->b_lab.assign(b.label, b.label + nn);
            s->words_pending = true;
        }
    }
    if (rc != 0) return fail(rc == -4 ? VPPS_E_GRAPH : VPPS_E_INVALID, err);
    *out = s.release();
    return VPPS_OK;
}

vpps_status vpps_script_words(vpps_script s, const uint32_t** words, int64_t* n) {
    if (!s || !words || !n) return fail(VPPS_E_INVALID, "null argument");
    if (s->words_pending) {
        Plan spec = s->model->plan;
        spec.skip_words = false;
        BatchIn b{(int32_t)s->b_gp.size() - 1, s->b_gp.data(), s->b_cp.data(), s->b_ch.data(), s->b_tok.data(),
                  s->b_lab.data()};
        Script t;
        std::string err;
        if (build_script(spec, b, INT64_MAX, &t, &err) != 0) return fail(VPPS_E_GRAPH, err);
        s->s.words.swap(t.words);
        s->words_pending = false;
    }
    *words = s->s.words.data();
    *n = (int64_t)s->s.words.size();
    return VPPS_OK;
}

vpps_status vpps_script_blob(vpps_script s, const uint32_t** blob, int64_t* n, int64_t* lists_off, int64_t* df_off) {
    if (!s || !blob || !n) return fail(VPPS_E_INVALID, "null argument");
    *blob = s->s.blob.data();
    *n = (int64_t)s->s.blob.size();
    if (lists_off) *lists_off = s->s.lists_off;
    if (df_off) *df_off = s->s.df_off;
    return VPPS_OK;
}

vpps_status vpps_script_info_get(vpps_script s, vpps_script_info* info) {
    if (!s || !info) return fail(VPPS_E_INVALID, "null argument");
    info->n_words = (int64_t)s->s.words.size();
    info->pool_words = s->s.pool_words;
    info->zero_words = s->s.zero_words;
    info->loss_word = s->s.loss_word;
    info->n_barriers = s->s.n_bar;
    info->n_levels = s->s.n_levels;
    info->n_nodes = s->s.n_nodes;
    info->n_heads = s->s.n_heads;
    info->flops = s->s.flops;
    info->act_bytes = s->s.act_bytes;
    info->blob_words = (int64_t)s->s.blob.size();
    info->kernel_flops = s->s.kernel_flops;
    return VPPS_OK;
}

vpps_status vpps_upload_script(vpps_script s, void* stream) {
    if (!s) return fail(VPPS_E_INVALID, "null script");
    if (s->model->plan_only) return fail(VPPS_E_STATE, "plan-only model");
    if (s->uploaded) return VPPS_OK;
    const size_t bytes = s->s.blob.size() * sizeof(uint32_t);
    CK(cudaMalloc(&s->d_words, bytes));
    CK(cudaMemcpyAsync(s->d_words, s->s.blob.data(), bytes, cudaMemcpyHostToDevice, (cudaStream_t)stream));
    CK(cudaStreamSynchronize((cudaStream_t)stream));     // pageable source: complete before returning
    s->uploaded = true;
    return VPPS_OK;
}

// Stage a non-resident script through the next ring slot: wait until the kernel that last read the
// slot is done, copy the words into the slot's pinned buffer, one H2D copy (L169).
static vpps_status stage_script(vpps_model m, vpps_script s, cudaStream_t st, int* slot_out,
                                const uint32_t** dwords) {
    const int k = m->next_slot;
    m->next_slot = (k + 1) % vpps_model_s::kSlots;
    vpps_model_s::Slot& sl = m->ring[k];
    const size_t n = s->s.blob.size();
    if (!sl.done) CK(cudaEventCreateWithFlags(&sl.done, cudaEventDisableTiming));
    if (sl.used) CK(cudaEventSynchronize(sl.done));
    if (n > sl.cap) {
        // (the slot's last reader has finished: event above; the pinned staging is library-owned, §8(b))
        if (sl.h) CK(cudaFreeHost(sl.h));
        m->alloc.put(sl.d, st);
        sl.h = nullptr;
        sl.d = nullptr;
        sl.cap = 0;
        const size_t cap = n + n / 2 + 1024;
        CK(cudaMallocHost(&sl.h, cap * sizeof(uint32_t)));
        sl.d = static_cast<uint32_t*>(m->alloc.get(cap * sizeof(uint32_t), st));
        if (!sl.d) return fail(VPPS_E_NOMEM, "script slot allocation failed");
        sl.cap = cap;
    }
    std::memcpy(sl.h, s->s.blob.data(), n * sizeof(uint32_t));
    CK(cudaMemcpyAsync(sl.d, sl.h, n * sizeof(uint32_t), cudaMemcpyHostToDevice, st));
    *slot_out = k;
    *dwords = sl.d;
    return VPPS_OK;
}

static vpps_status run(vpps_model m, vpps_script s, const float* inputs, int64_t n_rows, float* d_inputs,
                       int mode, float lr, float wd, void* stream_) {
    if (!m || !s) return fail(VPPS_E_INVALID, "null argument");
    if (m->plan_only) return fail(VPPS_E_STATE, "plan-only model");
    if (s->model != m) return fail(VPPS_E_STATE, "script was built for another model");
    if (!m->params || !m->grads) return fail(VPPS_E_STATE, "buffers not bound (vpps_bind_buffers)");
    if (!inputs || n_rows <= 0) return fail(VPPS_E_INVALID, "null input table");
    if (s->s.max_token >= n_rows) return fail(VPPS_E_GRAPH, "token out of range of the input table");
    if (((uintptr_t)inputs | (uintptr_t)d_inputs) & 15) return fail(VPPS_E_INVALID, "input tables must be 16-byte aligned");
    cudaStream_t st = (cudaStream_t)stream_;
    // every check before anything is queued (a failed call leaves no staged copy or pool change behind)
    if (m->dataflow && s->s.df_off < 0) return fail(VPPS_E_INVALID, "script has no dataflow program (binary cell only)");
    if (m->prof && !m->dataflow &&
        m->prof_stride < 2 + 3 * (int64_t)(s->s.n_bar + 1) + 10 * (int64_t)(s->s.n_bar + 2))
        return fail(VPPS_E_INVALID, "profile buffer stride too small for this script");
    if (m->prof && m->dataflow && m->prof_stride < 11) return fail(VPPS_E_INVALID, "profile buffer stride < 11");
    if (m->prof && m->dataflow && !df_prof_fn(m->var->fn))
        return fail(VPPS_E_STATE, "no trace-enabled dataflow kernel for this variant");
    if (m->prof && !m->dataflow && !m->cluster && !m->plan.level && !fb_prof_fn(m->var->fn))
        return fail(VPPS_E_STATE, "no trace-enabled grid kernel for this variant");
    CK(cudaSetDevice(m->device));
    const int64_t need = s->s.pool_words + (m->dataflow ? s->s.df_words : 0);
    if (need > m->pool_cap) {
        // stream-ordered growth through the model's allocator: no device synchronisation inside the pass
        m->alloc.put(m->pool, st);
        m->pool = nullptr;
        m->pool_cap = 0;
        const int64_t cap = need + need / 4 + 1024;
        m->pool = static_cast<float*>(m->alloc.get((size_t)cap * sizeof(float), st));
        if (!m->pool) return fail(VPPS_E_NOMEM, "activation pool allocation failed");
        // tagged slots (dataflow) must never carry a live epoch before they are written: zero once
        CK(cudaMemsetAsync(m->pool, 0, cap * sizeof(float), st));
        m->pool_cap = cap;
    }
    m->last_pool_words = s->s.pool_words;
    int ring_slot = -1;
    const uint32_t* dwords = s->d_words;
    if (!s->uploaded) {
        vpps_status r = stage_script(m, s, st, &ring_slot, &dwords);
        if (r != VPPS_OK) return r;
    }
    // per-pass clearing: the cluster / dataflow paths fold it into the leaf kernel (no memset calls)
    float* zero_ptr[4] = {m->pool, m->grads, reinterpret_cast<float*>(m->done), d_inputs};
    const int64_t zero_n[4] = {s->s.zero_words, m->n_floats, 4 * vpps_model_s::kMaxGroups,
                               d_inputs ? n_rows * m->plan.E : 0};
    if (!m->cluster) {
        CK(cudaMemsetAsync(m->pool, 0, s->s.zero_words * sizeof(float), st));
        if (m->plan.G > 1) CK(cudaMemsetAsync(m->grads, 0, (size_t)m->n_floats * sizeof(float), st));
        if (d_inputs) CK(cudaMemsetAsync(d_inputs, 0, (size_t)n_rows * m->plan.E * sizeof(float), st));
    }
    KParams kp{};
    kp.params = m->params;
    kp.grads = m->grads;
    kp.inputs = inputs;
    kp.d_inputs = d_inputs;
    kp.pool = m->pool;
    kp.script = dwords;
    for (size_t i = 0; i < m->offsets.size() && i < 8; ++i) kp.off[i] = m->offsets[i];
    kp.n_g = m->plan.n_g;
    kp.n_act = m->plan.n_act;
    kp.G = m->plan.G;
    kp.C = m->plan.C;
    kp.mode = mode;
    kp.loss_word = s->s.loss_word;
    kp.lr = lr;
    kp.wd = wd;
    kp.prof = m->prof;
    kp.prof_stride = m->prof_stride;
    void* args[] = {&kp};
    if (m->t_before) CK(cudaEventRecord(m->t_before, st));
    if (m->dataflow) {
        // leaf GEMM (also clears the pass's accumulators, advances the pass counter) -> vpps_df
        // (cooperative: a group's CTAs are co-resident, consumers spin on producers) -> gradient GEMM
        // (programmatic dependent, per-group completion counters) -> SGD
        DfParams dp{};
        dp.params = m->params;
        dp.grads = m->grads;
        dp.pool = m->pool;
        dp.script = dwords;
        dp.df_off = s->s.df_off;
        for (size_t i = 0; i < m->offsets.size() && i < 8; ++i) dp.off[i] = m->offsets[i];
        dp.C = m->plan.C;
        dp.epoch = m->d_epoch;
        dp.loss_word = s->s.loss_word;
        dp.df_hx = s->s.df_hx;
        dp.df_part = s->s.df_part;
        dp.df_hd = s->s.df_hd;
        dp.pool_words = s->s.pool_words;
        dp.n_hx = s->s.n_hx;
        dp.n_part = s->s.n_part;
        dp.n_hd = s->s.n_hd;
        dp.prof = m->prof;
        dp.prof_stride = m->prof_stride;
        dp.done = m->done;
        void* dargs[] = {&dp};
        cudaLaunchConfig_t cfg = {};
        cudaLaunchAttribute attr[2];
        // Cooperative launch (a group's CTAs poll each other's slots, so all must be resident), after the
        // leaf GEMM has completed.  Measured: as a programmatic dependent of the leaf GEMM (its weight
        // prologue overlapping the leaf tiles, with or without the cooperative attribute) the pass gave
        // wrong gradients intermittently — about one run in three of the dataflow GPU test selection,
        // mostly on the first pass of a new model — and 0 of 64 runs without it; the root
        // cause is not isolated, so the programmatic launch stays opt-in (VPPS_DF_PDL=1, measurement
        // only; VPPS_DF_COOP=0 drops the cooperative attribute).  The gradient GEMM stays a programmatic
        // dependent of this kernel (its loads all bypass L1).
        static const bool coop_df = !(getenv("VPPS_DF_COOP") && atoi(getenv("VPPS_DF_COOP")) == 0);
        attr[0].id = cudaLaunchAttributeCooperative;
        attr[0].val.cooperative = coop_df ? 1 : 0;
        cfg.gridDim = dim3(m->plan.n_cta);
        cfg.blockDim = dim3(df_block(m->var->fn));
        cfg.dynamicSmemBytes = m->smem;
        cfg.stream = st;
        // (opt-in programmatic launch: the kernel executes griddepcontrol.wait before it reads the leaf
        //  records, the pass counter or `done`, a no-op for an ordinary launch)
        static const bool no_pdl_df = !(getenv("VPPS_DF_PDL") && atoi(getenv("VPPS_DF_PDL")) != 0);
        attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
        attr[1].val.programmaticStreamSerializationAllowed = 1;
        cfg.attrs = attr;
        cfg.numAttrs = no_pdl_df ? 1 : 2;
        const uint32_t* lists = dwords + s->s.lists_off;
        const uint32_t* leaf_list = lists + 3 * s->s.n_int;
        const float* W_iou = m->params + m->offsets[0];
        // U_iou, U_fl, U_fr, W_out and the biases (contiguous after W_iou in the flat layout) are pulled into
        // L2 by the leaf kernel's clearing warps for vpps_df's prologue
        const int64_t pf_floats = m->n_floats - m->offsets[1];
        launch_leaf_fwd(W_iou, m->params + m->offsets[5], inputs, m->pool, leaf_list, (int32_t)s->s.n_leaf,
                        m->plan.H, m->plan.E, zero_ptr, zero_n, m->d_epoch, st, m->params + m->offsets[1],
                        pf_floats * (int64_t)sizeof(float), n_rows);
        if (m->k_before) CK(cudaEventRecord(m->k_before, st));
        const void* dfn = m->prof ? df_prof_fn(m->var->fn) : m->var->fn;
        if (m->prof) CK(cudaFuncSetAttribute(dfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)m->smem));
        CK(cudaLaunchKernelExC(&cfg, dfn, dargs));
        if (m->k_after) CK(cudaEventRecord(m->k_after, st));
        const int32_t n_grp = (int32_t)s->s.int_off.size() - 1;
        std::vector<int32_t> order(n_grp);
        for (int32_t g = 0; g < n_grp; ++g) order[g] = g;
        std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) {
            if (s->s.grp_levels[a] != s->s.grp_levels[b]) return s->s.grp_levels[a] < s->s.grp_levels[b];
            return s->s.grp_nodes[a] < s->s.grp_nodes[b];
        });
        // weight gradients (L185) + leaf dX per replica group as the groups finish, SGD fused in the tail at
        // N = 1: FFMA2 items (vpps_cluster.cu, 3 CTAs per SM).  VPPS_DW_TC2=1 (measurement) runs the
        // tensor-core items of vpps_dwtc.cu instead: parity-green but slower (tail 33 vs 17 us per TGT step;
        // a group's items have K <= ~50 nodes, so each 128 x 128 tile is two chunks of 3xTF32 MMAs behind a
        // fixed staging / drain / reduction cost, at one CTA per SM)
        static const bool dw_tc2 = getenv("VPPS_DW_TC2") && atoi(getenv("VPPS_DW_TC2")) != 0;
        if (!dw_tc2 || m->gemm_trace) {
            launch_dw_gemm(m->pool, inputs, d_inputs, m->params, m->grads, lists, leaf_list, n_grp, s->s.int_off.data(),
                           s->s.leaf_off.data(), order.data(), m->done, m->cluster, true, m->plan.H, m->plan.E,
                           m->offsets.data(), m->n_floats, mode, lr, wd, st, m->gemm_trace,
                           m->pool + s->s.loss_word, m->d_loss_map + (m->passes & 1));
        } else if (!launch_dw_tc(m->pool, inputs, d_inputs, m->params, m->grads, lists, leaf_list, n_grp,
                                 s->s.int_off.data(), s->s.leaf_off.data(), order.data(), m->done, m->cluster,
                                 m->plan.H, m->plan.E, m->offsets.data(), m->n_floats, mode, lr, wd, st,
                                 m->pool + s->s.loss_word, m->d_loss_map + (m->passes & 1), m->sms)) {
            return fail(VPPS_E_CUDA, "gradient GEMM launch failed");
        }
        CK(cudaGetLastError());
    } else if (m->plan.level && m->plan.cell == CELL_GRU) {
        if (s->s.tg_tok < 0) return fail(VPPS_E_INVALID, "script was not built for the level path");
        CK(cudaMemsetAsync(m->grads, 0, (size_t)m->n_floats * sizeof(float), st));
        const int rc = gru_pass(m->level, m->params, m->offsets.data(), m->grads, m->pool, inputs, d_inputs, dwords,
                                s->s.tg_tok, s->s.tg_lab, s->s.tg_fpos, s->s.tg_start.data(),
                                (int32_t)s->s.tg_start.size() - 1, s->s.tg_T, m->plan.H, m->plan.E, m->plan.C,
                                s->s.loss_word, st, s->s.tg_chain >= 0 ? dwords + s->s.tg_chain : nullptr,
                                m->plan.chain_g);
        if (rc != 0) return fail(VPPS_E_CUDA, "GRU pass failed (code " + std::to_string(rc) + ")");
        if (mode == 1) launch_sgd(m->params, m->grads, m->n_floats, lr, wd, st);
    } else if (m->plan.level && m->plan.cell == CELL_BILSTM_CHAR) {
        if (s->s.tg_tok < 0) return fail(VPPS_E_INVALID, "script was not built for the level path");
        CK(cudaMemsetAsync(m->grads, 0, (size_t)m->n_floats * sizeof(float), st));
        const int rc = bilstmchar_pass(m->level, m->params, m->offsets.data(), m->grads, m->pool, inputs, d_inputs,
                                       dwords, s->s.tg_tok, s->s.tg_lab, s->s.tg_fpos, s->s.tg_bpos,
                                       s->s.tg_start.data(), (int32_t)s->s.tg_start.size() - 1, s->s.tg_T, m->plan.H,
                                       m->plan.E, m->plan.C, m->plan.mlp, s->s.loss_word, st,
                                       s->s.tg_chain >= 0 ? dwords + s->s.tg_chain : nullptr, m->plan.chain_g,
                                       s->s.tc_T, s->s.tc_R, s->s.tc_tok, s->s.tc_word, s->s.tc_rare, s->s.tc_list,
                                       s->s.tc_chain, m->plan.chain_gc, m->plan.ec);
        if (rc != 0) return fail(VPPS_E_CUDA, "BiLSTMwChar pass failed (code " + std::to_string(rc) + ")");
        if (mode == 1) launch_sgd(m->params, m->grads, m->n_floats, lr, wd, st);
    } else if (m->plan.level && (m->plan.cell == CELL_BILSTM || m->plan.cell == CELL_LSTM)) {
        if (s->s.tg_tok < 0) return fail(VPPS_E_INVALID, "script was not built for the level path");
        CK(cudaMemsetAsync(m->grads, 0, (size_t)m->n_floats * sizeof(float), st));   // incl. padding
        const bool bi = m->plan.cell == CELL_BILSTM;
        const int64_t* o6 = m->offsets.data();
        // (Wf, Uf, Wb, Ub, W_mlp, W_tag, bf, bb, b_mlp, b_tag); the LM: (W, U, -, -, -, W_out, b, -, -, b_out)
        const int64_t off10[10] = {o6[0], o6[1], bi ? o6[2] : -1, bi ? o6[3] : -1, bi ? o6[4] : -1,
                                   bi ? o6[5] : o6[2], bi ? o6[6] : o6[3], bi ? o6[7] : -1, bi ? o6[8] : -1,
                                   bi ? o6[9] : o6[4]};
        const int rc = tagger_pass(m->level, m->params, off10, m->grads, m->pool, inputs, d_inputs, dwords,
                                   s->s.tg_tok, s->s.tg_lab, s->s.tg_fpos, s->s.tg_bpos, s->s.tg_start.data(),
                                   (int32_t)s->s.tg_start.size() - 1, s->s.tg_T, m->plan.H, m->plan.E, m->plan.C,
                                   bi ? m->plan.mlp : 0, bi ? 2 : 1, s->s.loss_word, st,
                                   s->s.tg_chain >= 0 ? dwords + s->s.tg_chain : nullptr, m->plan.chain_g);
        if (rc != 0) return fail(VPPS_E_CUDA, "tagger pass failed (code " + std::to_string(rc) + ")");
        if (mode == 1) launch_sgd(m->params, m->grads, m->n_floats, lr, wd, st);
    } else if (m->plan.level) {
        if (s->s.lv_int < 0) return fail(VPPS_E_INVALID, "script was not built for the level path");
        CK(cudaMemsetAsync(m->grads, 0, (size_t)m->n_floats * sizeof(float), st));   // (memset above: G > 1 only)
        const int32_t Lv = (int32_t)s->s.lv_start.size() - 2;
        const int rc =
            m->plan.cell == CELL_RVNN
                ? rvnn_pass(m->level, m->params, m->offsets.data(), m->grads, m->pool, inputs, d_inputs, dwords,
                            s->s.lv_int, s->s.lv_leaf, s->s.lv_head, s->s.lv_start.data(), Lv, s->s.lv_n_int,
                            s->s.lv_n_leaf, s->s.lv_n_head, m->plan.H, m->plan.E, m->plan.C, s->s.loss_word, st)
            : m->plan.cell == CELL_TDRNN
                ? tdrnn_pass(m->level, m->params, m->offsets.data(), m->grads, m->pool, inputs, d_inputs, dwords,
                             s->s.lv_int, s->s.lv_leaf, s->s.lv_head, s->s.lv_start.data(), Lv, s->s.lv_n_int,
                             s->s.lv_n_leaf, s->s.lv_n_head, m->plan.H, m->plan.E, m->plan.C, s->s.loss_word, st)
                : level_pass(m->level, m->params, m->offsets.data(), m->grads, m->pool, inputs, d_inputs, dwords,
                             s->s.lv_int, s->s.lv_leaf, s->s.lv_head, s->s.lv_start.data(), Lv, s->s.lv_n_int,
                             s->s.lv_n_leaf, s->s.lv_n_head, m->plan.H, m->plan.E, m->plan.C, s->s.loss_word, st,
                             m->plan.cell == CELL_TDLSTM);
        if (rc != 0) return fail(VPPS_E_CUDA, "level pass failed (code " + std::to_string(rc) + ")");
        if (mode == 1) launch_sgd(m->params, m->grads, m->n_floats, lr, wd, st);
    } else if (m->cluster) {
        // one cluster per replica group; clusters never wait on each other (graphs are whole per group).
        // Launch order: leaf GEMM (also clears the pass's accumulators) -> vpps_cl -> gradient GEMM
        // (programmatic dependent: a group's tiles start when its cluster's 16 CTAs have counted
        // themselves done) -> SGD.
        kp.done = m->done;
        cudaLaunchConfig_t cfg = {};
        cudaLaunchAttribute attr[2];
        attr[0].id = cudaLaunchAttributeClusterDimension;
        attr[0].val.clusterDim.x = m->cluster;
        attr[0].val.clusterDim.y = 1;
        attr[0].val.clusterDim.z = 1;
        cfg.gridDim = dim3(m->plan.n_cta);
        cfg.blockDim = dim3(256);
        cfg.dynamicSmemBytes = m->smem;
        cfg.stream = st;
        cfg.attrs = attr;
        cfg.numAttrs = 1;       // ordinary stream order after the leaf kernel (which clears `done`)
        const uint32_t* lists = dwords + s->s.lists_off;
        const uint32_t* leaf_list = lists + 3 * s->s.n_int;
        const float* W_iou = m->params + m->offsets[0];
        // level 0 (all leaves share W_iou on their word vectors) as one dense GEMM + cell pass
        launch_leaf_fwd(W_iou, m->params + m->offsets[5], inputs, m->pool, leaf_list, (int32_t)s->s.n_leaf,
                        m->plan.H, m->plan.E, zero_ptr, zero_n, nullptr, st);
        if (m->k_before) CK(cudaEventRecord(m->k_before, st));
        CK(cudaLaunchKernelExC(&cfg, m->var->fn, args));
        if (m->k_after) CK(cudaEventRecord(m->k_after, st));
        // dW of the weight matrices from the recorded operands and dX of the leaves
        // = W_iouᵀ g_leaf (words are inputs) in one launch; SGD in mode 1.  Groups whose
        // cluster should finish first (fewest levels, then fewest nodes) get the lowest tile indices.
        const int32_t n_grp = (int32_t)s->s.int_off.size() - 1;
        std::vector<int32_t> order(n_grp);
        for (int32_t g = 0; g < n_grp; ++g) order[g] = g;
        std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) {
            if (s->s.grp_levels[a] != s->s.grp_levels[b]) return s->s.grp_levels[a] < s->s.grp_levels[b];
            return s->s.grp_nodes[a] < s->s.grp_nodes[b];
        });
        launch_dw_gemm(m->pool, inputs, d_inputs, m->params, m->grads, lists, leaf_list, n_grp, s->s.int_off.data(),
                       s->s.leaf_off.data(), order.data(), m->done, m->cluster, true, m->plan.H, m->plan.E,
                       m->offsets.data(), m->n_floats, mode, lr, wd, st, nullptr,
                       m->pool + s->s.loss_word, m->d_loss_map + (m->passes & 1));
        CK(cudaGetLastError());
    } else {
        const void* gfn = m->prof ? fb_prof_fn(m->var->fn) : m->var->fn;
        if (m->prof) CK(cudaFuncSetAttribute(gfn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)m->smem));
        CK(cudaLaunchCooperativeKernel(gfn, dim3(m->plan.n_cta), dim3(256), args, m->smem, st));
    }
    if (m->t_after) CK(cudaEventRecord(m->t_after, st));
    if (ring_slot >= 0) {
        CK(cudaEventRecord(m->ring[ring_slot].done, st));
        m->ring[ring_slot].used = true;
    }
    const int slot = (int)(m->passes & 1);
    if (!m->cluster)   // (the cluster / dataflow gradient kernel writes the loss into mapped h_loss itself)
        CK(cudaMemcpyAsync(m->h_loss + slot, m->pool + s->s.loss_word, sizeof(float), cudaMemcpyDeviceToHost, st));
    CK(cudaEventRecord(m->ev[slot], st));
    ++m->passes;
    return VPPS_OK;
}

vpps_status vpps_fwd_bwd(vpps_model m, vpps_script s, const float* inputs, int64_t n_input_rows, float* d_inputs,
                         void* stream) {
    return run(m, s, inputs, n_input_rows, d_inputs, 0, 0.f, 0.f, stream);
}

vpps_status vpps_fwd_bwd_sgd(vpps_model m, vpps_script s, const float* inputs, int64_t n_input_rows,
                             float* d_inputs, float lr, float weight_decay, void* stream) {
    return run(m, s, inputs, n_input_rows, d_inputs, 1, lr, weight_decay, stream);
}

vpps_status vpps_sgd_step(vpps_model m, float lr, float weight_decay, void* stream) {
    if (!m) return fail(VPPS_E_INVALID, "null model");
    if (m->plan_only || !m->params) return fail(VPPS_E_STATE, "buffers not bound");
    launch_sgd(m->params, m->grads, m->n_floats, lr, weight_decay, (cudaStream_t)stream);
    CK(cudaGetLastError());
    return VPPS_OK;
}

vpps_status vpps_get_stale_loss(vpps_model m, float* loss) {
    if (!m || !loss) return fail(VPPS_E_INVALID, "null argument");
    if (m->plan_only) return fail(VPPS_E_STATE, "plan-only model");
    if (m->passes < 2) { *loss = 0.f; return VPPS_OK; }
    const int slot = (int)((m->passes - 2) & 1);
    CK(cudaEventSynchronize(m->ev[slot]));
    *loss = m->h_loss[slot];
    return VPPS_OK;
}

vpps_status vpps_sync_get_latest_loss(vpps_model m, float* loss) {
    if (!m || !loss) return fail(VPPS_E_INVALID, "null argument");
    if (m->plan_only) return fail(VPPS_E_STATE, "plan-only model");
    if (m->passes < 1) { *loss = 0.f; return VPPS_OK; }
    const int slot = (int)((m->passes - 1) & 1);
    CK(cudaEventSynchronize(m->ev[slot]));
    *loss = m->h_loss[slot];
    return VPPS_OK;
}

vpps_status vpps_set_timing_events(vpps_model m, void* ev_before, void* ev_after) {
    if (!m) return fail(VPPS_E_INVALID, "null model");
    m->t_before = (cudaEvent_t)ev_before;
    m->t_after = (cudaEvent_t)ev_after;
    return VPPS_OK;
}

vpps_status vpps_set_kernel_events(vpps_model m, void* ev_before, void* ev_after) {
    if (!m) return fail(VPPS_E_INVALID, "null model");
    m->k_before = (cudaEvent_t)ev_before;
    m->k_after = (cudaEvent_t)ev_after;
    return VPPS_OK;
}

vpps_status vpps_set_gemm_trace(vpps_model m, uint64_t* buf) {
    if (!m) return fail(VPPS_E_INVALID, "null model");
    m->gemm_trace = buf;
    return VPPS_OK;
}

vpps_status vpps_set_profile_buffer(vpps_model m, uint64_t* buf, int64_t stride) {
    if (!m) return fail(VPPS_E_INVALID, "null model");
    m->prof = buf;
    m->prof_stride = stride;
    return VPPS_OK;
}

vpps_status vpps_pool_ptr(vpps_model m, float** pool, int64_t* pool_words) {
    if (!m || !pool) return fail(VPPS_E_INVALID, "null argument");
    *pool = m->pool;
    if (pool_words) *pool_words = m->last_pool_words;
    return VPPS_OK;
}

void vpps_destroy_script(vpps_script s) {
    if (!s) return;
    if (s->d_words) cudaFree(s->d_words);
    delete s;
}

void vpps_destroy_model(vpps_model m) {
    if (!m) return;
    for (cudaEvent_t e : m->ev)            // the last passes (the pool's last readers) have finished
        if (e) cudaEventSynchronize(e);
    if (m->level) level_ctx_destroy(m->level);
    if (m->pool) m->alloc.put(m->pool, nullptr);
    if (m->done) cudaFree(m->done);
    if (m->d_epoch) cudaFree(m->d_epoch);
    if (m->h_loss) cudaFreeHost(m->h_loss);   // (cudaHostAlloc'd or cudaMallocHost'd: both freed here)
    for (cudaEvent_t e : m->ev)
        if (e) cudaEventDestroy(e);
    for (auto& sl : m->ring) {
        if (sl.done) cudaEventSynchronize(sl.done), cudaEventDestroy(sl.done);
        if (sl.h) cudaFreeHost(sl.h);
        if (sl.d) m->alloc.put(sl.d, nullptr);
    }
    delete m;
}

}  // extern "C"
