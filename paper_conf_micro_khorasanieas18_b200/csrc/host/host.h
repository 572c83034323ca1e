// Host-side data structures of libvpps (partition plan, super-graph, script).
// Written from SPEC_SCRIPT.md; PAPER.md line citations at each function.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

namespace vpps {

constexpr uint32_t NONE = 0xFFFFFFFFu;

enum Cell : int32_t { CELL_LSTM = 0, CELL_BINARY = 1, CELL_CHILDSUM = 2, CELL_BILSTM = 3, CELL_GRU = 4, CELL_RVNN = 5, CELL_TDRNN = 6, CELL_TDLSTM = 7, CELL_BILSTM_CHAR = 8 };

enum Op : uint32_t {
    OP_S = 0x01, OP_W = 0x02,
    OP_LSTM_F = 0x10, OP_LSTM_B = 0x11,
    OP_LEAF_F = 0x20, OP_LEAF_B = 0x21, OP_INT_F = 0x22, OP_INT_B = 0x23,
    OP_CS_F = 0x30, OP_CS_B = 0x31,
    OP_HEAD_F = 0x40, OP_HEAD_B = 0x41, OP_HEAD_FB = 0x42,   // HEAD_FB: dataflow program only
};

struct Shape { int32_t rows, cols; };

// ---- SPEC P0: paper-literal dealer --------------------------------------------------------
struct DealRow { int32_t matrix, row, cta, partition, warp, is_grad; };
int32_t regs_per_row(int32_t row_max);
int32_t reg_budget(int32_t tb, int32_t cps);
void paper_deal(const std::vector<Shape>& mats, int32_t n_cta, int32_t tb, int32_t rpw, bool pack_rows,
                bool grads, std::vector<DealRow>* rows, int64_t* n_slots);
int32_t paper_choose_cps(const std::vector<Shape>& mats, int32_t n_sm, int32_t tb, int32_t rpw, bool pack_rows);

// ---- SPEC P1: unit-bundle plan --------------------------------------------------------------
struct Plan {
    int32_t cell, H, E, C;
    int32_t mlp = 0;         // BiLSTM tagger MLP width (256)
    int32_t n_cta, n_g, n_act, umax, G;
    bool by_graph = false;   // SPEC S5g: whole graphs assigned to groups (cluster replicas)
    bool level = false;      // level-synchronous GEMM path (binary cell, weights L2-resident)
    int32_t vc = 0, ec = 0;  // BiLSTMwChar: characters and character-embedding width (C_emb is Vc x Ec)
    int32_t chain_gc = 0;    // BiLSTMwChar: chain groups per direction of the character recurrence (H_c = E/2)
    int32_t chain_g = 0;     // chain cells on the level path: groups per direction of the register-resident
                             // recurrence (vpps_chain.cu); 0 = per-step products
    bool skip_words = false; // dataflow models: the SPEC words (S4-S6, §E) are not built with the device
                             // lowering (its kernels never read them); vpps_script_words builds them on demand
    std::vector<int32_t> table;   // rows of 8 int32
};
bool unit_plan(int32_t cell, int32_t H, int32_t E, int32_t C, int32_t n_sm, int32_t cps, int32_t G,
               Plan* out, std::string* err);

// ---- SPEC §S/§E: script ----------------------------------------------------------------------
struct BatchIn {
    int32_t n_graphs;
    const int32_t* graph_ptr;
    const int32_t* child_ptr;
    const int32_t* children;
    const int32_t* token;
    const int32_t* label;
    const int32_t* char_ptr = nullptr;   // BiLSTMwChar spellings (CSR over the nodes) or nullptr
    const int32_t* chars = nullptr;
};

struct Script {
    std::vector<uint32_t> words;
    int64_t pool_words = 0, zero_words = 0, loss_word = 0;
    int32_t n_bar = 0, n_levels = 0;
    int64_t n_nodes = 0, n_heads = 0, max_token = -1;
    // device upload blob = words ‖ (rec, rec_l, rec_r) per internal node ‖ (rec, token) per leaf; the node
    // lists drive the gradient GEMM of the cluster path.  Not part of the SPEC words.
    std::vector<uint32_t> blob;
    int64_t lists_off = 0;   // blob offset of the INT list (= words.size(), 0 when the words are skipped)
    int64_t n_int = 0, n_leaf = 0;
    // per replica group g (S5g plans; one group otherwise): its internal / leaf nodes are list entries
    // [int_off[g], int_off[g+1]) / [leaf_off[g], leaf_off[g+1]); node count and deepest level
    std::vector<int32_t> int_off, leaf_off, grp_nodes, grp_levels;
    // dataflow program of the binary cell for whole-graph groups (vpps_df): blob word offset (-1: none),
    // tagged-slot counts and their pool word offsets (regions behind pool_words, df_words long)
    int64_t df_off = -1, n_hx = 0, n_part = 0, n_hd = 0;
    int64_t df_hx = 0, df_part = 0, df_hd = 0, df_words = 0;
    double flops = 0.0, act_bytes = 0.0;
    double kernel_flops = 0.0;   // binary whole-graph paths: FLOPs of the replica-group kernel alone
    // level-synchronous path (Plan::level): blob word offsets of the internal-node list sorted by level
    // (rec, rec_l, rec_r, adj, adj_l, adj_r), the leaf list (rec, adj, token) and the head list
    // (rec, rec_c, adj_c, label); lv_start[l] = first internal node of level l (l = 1 .. L+1)
    int64_t lv_int = -1, lv_leaf = -1, lv_head = -1;
    int64_t lv_n_int = 0, lv_n_leaf = 0, lv_n_head = 0;
    std::vector<int32_t> lv_start;
    // BiLSTM tagger (CELL_BILSTM, level path): T positions (sentences concatenated), blob offsets of
    // tok[T], lab[T], the forward step lists fpos[T] (positions of step t: sentences longer than t, in
    // batch order, starting at fstart[t]) and the backward step lists bpos[T] (position len-1-t)
    int64_t tg_T = 0, tg_tok = -1, tg_lab = -1, tg_fpos = -1, tg_bpos = -1;
    int64_t tg_chain = -1;           // blob offset of the chain-recurrence sentence table (SPEC §L), or -1
    // BiLSTMwChar (SPEC §L): R rare positions, Tc character positions (spellings concatenated in position
    // order); blob offsets of ctok[Tc] (character ids), cword[Tc] (rare index of each character position),
    // rare[T] (rare index of a word position or NONE), rlist[R][3] (word position, character offset,
    // length) and the character chain table
    int64_t tc_T = 0, tc_R = 0, tc_tok = -1, tc_word = -1, tc_rare = -1, tc_list = -1, tc_chain = -1;
    std::vector<int32_t> tg_start;   // [maxlen + 1]
};

// Returns 0 on success, -4 (graph error) or -1 (invalid) with a message.
int build_script(const Plan& plan, const BatchIn& b, int64_t n_input_rows, Script* out, std::string* err);
// BiLSTM tagger batches (chains: node t has child t-1 and a token; labels are tags < C).
int build_tagger_script(const Plan& plan, const BatchIn& b, int64_t n_input_rows, Script* out, std::string* err);

}  // namespace vpps
