// Per-batch script generation (SPEC_SCRIPT.md §S, §E).
//
// PAPER.md §III-B1: super-graph with aggregated loss (L205); nodes sorted by maximum depth from the
// sources (L139); forward traversal level by level emitting one CISC instruction per node (L141,
// L159: 4-byte preamble with op type and input tensor length, then 4-byte pool offsets); signal and
// wait between consecutive levels among the participating virtual processors (L165); reverse
// traversal for back-propagation with min-load assignment (L167); scripts concatenated behind the
// prefix sum of their lengths for one host-to-device copy (L169).
#include <algorithm>
#include <cstring>
#include "host.h"
#ifdef VPPS_HOST_PHASES   // measurement build (tools/host_breakdown.py): per-phase host times
#include <chrono>
double vpps_host_phase_us[8];
#define PHASE(k) do { const double _n = std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now().time_since_epoch()).count(); if (k > 0) vpps_host_phase_us[k - 1] += _n - _t0; _t0 = _n; } while (0)
#else
#define PHASE(k) do { } while (0)
#endif

namespace vpps {
namespace {

inline int64_t align32(int64_t x) { return (x + 31) / 32 * 32; }
inline uint32_t preamble(uint32_t op, int64_t len) { return op | (uint32_t)(len << 8); }

enum Kind : int8_t { K_LEAF, K_INT, K_CS, K_LSTM, K_HEAD };

struct Node {
    Kind kind;
    int32_t token, label;
    int32_t ch_begin, ch_count;   // into Graph::kids (global ids)
    int32_t graph;
};

}  // namespace

int build_script(const Plan& plan, const BatchIn& b, int64_t n_input_rows, Script* out, std::string* err) {
    const int64_t H = plan.H, E = plan.E, C = plan.C;
    if (b.n_graphs < 0 || (b.n_graphs > 0 && (!b.graph_ptr || !b.child_ptr || !b.token || !b.label))) {
        *err = "null batch array";
        return -1;
    }
#ifdef VPPS_HOST_PHASES
    double _t0 = 0;
#endif
    PHASE(0);
    // ---- S1/S2: super-graph (cells in given order, then heads of labelled cells) -----------------
    std::vector<Node> nodes;
    std::vector<int32_t> kids;
    std::vector<int32_t> parents_seen;
    for (int32_t g = 0; g < b.n_graphs; ++g) {
        const int32_t first = b.graph_ptr[g], last = b.graph_ptr[g + 1];
        if (last < first) { *err = "graph_ptr not monotone"; return -4; }
        const int32_t base = (int32_t)nodes.size();
        parents_seen.assign(last - first, 0);
        for (int32_t v = first; v < last; ++v) {
            const int32_t local = v - first;
            const int32_t c0 = b.child_ptr[v], c1 = b.child_ptr[v + 1];
            const int32_t nch = c1 - c0, tok = b.token[v], lab = b.label[v];
            if (nch < 0) { *err = "child_ptr not monotone"; return -4; }
            if (tok < -1 || tok >= n_input_rows) { *err = "token out of range"; return -4; }
            if (lab < -1 || lab >= C) { *err = "label out of range"; return -4; }
            Node nd{K_CS, tok, lab, (int32_t)kids.size(), nch, g};
            for (int32_t k = c0; k < c1; ++k) {
                const int32_t ch = b.children[k];
                if (ch < 0 || ch >= local) { *err = "children must precede their parent"; return -4; }
                if (++parents_seen[ch] > 1 && plan.cell != CELL_TDRNN && plan.cell != CELL_TDLSTM) {   // TD DAGs (R-36/37)
                    *err = "a node may have at most one parent";
                    return -4;
                }
                kids.push_back(base + ch);
            }
            switch (plan.cell) {
                case CELL_RVNN:
                case CELL_TDRNN:
                case CELL_TDLSTM:
                case CELL_BINARY:
                    if (nch == 0 && tok >= 0) nd.kind = K_LEAF;
                    else if (nch == 2 && tok < 0) nd.kind = K_INT;
                    else { *err = "binary Tree-LSTM: leaves carry a token, internal nodes have 2 children"; return -4; }
                    break;
                case CELL_LSTM:
                    if (nch > 1 || tok < 0 || (nch == 1 && b.children[c0] != local - 1)) {
                        *err = "LSTM chain: node t has child t-1 and a token";
                        return -4;
                    }
                    nd.kind = K_LSTM;
                    break;
                default:
                    if (nch > 8) { *err = "child-sum node with more than 8 children"; return -4; }
                    nd.kind = K_CS;
            }
            nodes.push_back(nd);
        }
        for (int32_t v = first; v < last; ++v)
            if (b.label[v] >= 0) {
                nodes.push_back(Node{K_HEAD, -1, b.label[v], (int32_t)kids.size(), 1, g});
                kids.push_back(base + (v - first));
            }
    }
    const int64_t N = (int64_t)nodes.size();
    if (N == 0) { *err = "empty batch"; return -4; }

    PHASE(1);
    // ---- S3: level = maximum depth from the sources (L139) --------------------------------------
    std::vector<int32_t> level(N, 0);
    int32_t L = 0;
    for (int64_t i = 0; i < N; ++i) {
        int32_t lv = 0;
        for (int32_t k = 0; k < nodes[i].ch_count; ++k)
            lv = std::max(lv, level[kids[nodes[i].ch_begin + k]] + 1);
        level[i] = lv;
        L = std::max(L, lv);
    }

    // ---- S7: pool plan ------------------------------------------------------------------------
    const int32_t n_bar = 2 * L + 1;
    const int64_t loss_word = align32(n_bar + 1);
    int64_t cursor = align32(loss_word + 1);
    std::vector<uint32_t> adj(N, NONE), rec(N, 0);
    for (int64_t i = 0; i < N; ++i)
        if (nodes[i].kind != K_HEAD) { adj[i] = (uint32_t)cursor; cursor = align32(cursor + 2 * H); }
    const int64_t zero_words = cursor;
    for (int64_t i = 0; i < N; ++i) {
        int64_t sz = 0;
        switch (nodes[i].kind) {
            case K_LSTM: sz = (6 + 4) * H; break;          // forward fields + gate gradients (§S7)
            case K_LEAF: sz = (5 + 3) * H; break;
            case K_INT: sz = (7 + 5) * H; break;
            case K_CS: sz = (8 + 2 * nodes[i].ch_count) * H; break;
            case K_HEAD: sz = C + 1; break;
        }
        rec[i] = (uint32_t)cursor;
        cursor = align32(cursor + sz);
    }
    if (cursor >= (int64_t)NONE) { *err = "pool exceeds 2^32 words (16 GiB, L159)"; return -1; }

    PHASE(2);
    // ---- per-node cost (MACs; L167 "relatively higher load" for cached-matrix ops) and FLOPs -----
    auto macs = [&](int64_t i) -> int64_t {
        const Node& n = nodes[i];
        switch (n.kind) {
            case K_LEAF: return 3 * H * E;
            case K_INT: return 8 * H * H;
            case K_CS: return (n.token >= 0 ? 4 * H * E : 0) + (n.ch_count ? (3 + n.ch_count) * H * H : 0);
            case K_LSTM: return 4 * H * E + (n.ch_count ? 4 * H * H : 0);
            case K_HEAD: return C * H;
        }
        return 0;
    };
    double flops = 0.0, abytes = 0.0;
    for (int64_t i = 0; i < N; ++i) {
        if (plan.cell == CELL_RVNN)       // M6: leaf H×E, internal H×2H, head C×H
            flops += 6.0 * (double)(nodes[i].kind == K_LEAF ? H * E : nodes[i].kind == K_INT ? 2 * H * H : C * H);
        else if (plan.cell == CELL_TDRNN)   // M7: no leaf transform, inner H×2H, head C×H
            flops += 6.0 * (double)(nodes[i].kind == K_LEAF ? 0 : nodes[i].kind == K_INT ? 2 * H * H : C * H);
        else
            flops += 6.0 * (double)macs(i);   // forward, weight gradient, input/hidden gradient (2 FLOP/MAC)
        const Node& n = nodes[i];
        const double nc = n.ch_count;
        double kin = 0, recsz = 0;
        switch (n.kind) {
            case K_LEAF: kin = E; recsz = 5 * H; break;
            case K_INT: kin = 2 * H; recsz = 7 * H; break;
            case K_CS: kin = E + H * (1 + nc); recsz = (5 + nc) * H; break;
            case K_LSTM: kin = E + H; recsz = 6 * H; break;
            case K_HEAD: kin = H; recsz = C + 1; break;
        }
        if (n.kind == K_HEAD) abytes += 4.0 * (H + (C + 1) + (C + 1) + 2 * H);
        else abytes += 4.0 * ((kin + nc * H + recsz) + (recsz + 2 * H + kin + nc * H + nc * 2 * H));
    }

    // ---- instruction encoding (§E) -------------------------------------------------------------
    auto emit = [&](std::vector<uint32_t>& w, int64_t i, bool fwd) {
        const Node& n = nodes[i];
        const int32_t* ch = kids.data() + n.ch_begin;
        const uint32_t tok = n.token < 0 ? NONE : (uint32_t)n.token;
        switch (n.kind) {
            case K_LEAF:
                if (fwd) w.insert(w.end(), {preamble(OP_LEAF_F, E), rec[i], tok});
                else w.insert(w.end(), {preamble(OP_LEAF_B, E), rec[i], adj[i], tok});
                break;
            case K_INT:
                if (fwd) w.insert(w.end(), {preamble(OP_INT_F, 2 * H), rec[i], rec[ch[0]], rec[ch[1]]});
                else w.insert(w.end(), {preamble(OP_INT_B, 2 * H), rec[i], adj[i], rec[ch[0]], adj[ch[0]],
                                        rec[ch[1]], adj[ch[1]]});
                break;
            case K_LSTM: {
                const uint32_t pr = n.ch_count ? rec[ch[0]] : NONE, pa = n.ch_count ? adj[ch[0]] : NONE;
                if (fwd) w.insert(w.end(), {preamble(OP_LSTM_F, E + H), rec[i], tok, pr});
                else w.insert(w.end(), {preamble(OP_LSTM_B, E + H), rec[i], adj[i], tok, pr, pa});
                break;
            }
            case K_CS:
                if (fwd) {
                    w.insert(w.end(), {preamble(OP_CS_F, n.ch_count), rec[i], tok});
                    for (int32_t k = 0; k < n.ch_count; ++k) w.push_back(rec[ch[k]]);
                } else {
                    w.insert(w.end(), {preamble(OP_CS_B, n.ch_count), rec[i], adj[i], tok});
                    for (int32_t k = 0; k < n.ch_count; ++k) { w.push_back(rec[ch[k]]); w.push_back(adj[ch[k]]); }
                }
                break;
            case K_HEAD:
                if (fwd) w.insert(w.end(), {preamble(OP_HEAD_F, H), rec[i], rec[ch[0]], (uint32_t)n.label});
                else w.insert(w.end(), {preamble(OP_HEAD_B, H), rec[i], rec[ch[0]], adj[ch[0]], (uint32_t)n.label});
                break;
        }
    };

    PHASE(3);
    // ---- S4-S6: phases, min-load groups, signal/wait ------------------------------------------
    const int32_t G = plan.G, P = 2 * L + 2;
    std::vector<std::vector<int64_t>> at_level(L + 1);
    // S4 (reading R-13): cells before heads, each in ascending global id — consecutive same-opcode
    // instructions form one batch in the kernels (an LM level alternates cell / head otherwise)
    for (int64_t i = 0; i < N; ++i)
        if (nodes[i].kind != K_HEAD) at_level[level[i]].push_back(i);
    for (int64_t i = 0; i < N; ++i)
        if (nodes[i].kind == K_HEAD) at_level[level[i]].push_back(i);
    std::vector<std::vector<uint32_t>> streams(G);
    std::vector<uint32_t> targets(n_bar + 1, 0);
    std::vector<std::vector<uint32_t>> body(G);
    std::vector<int64_t> load(G);
    std::vector<char> was_active(G, 0);
    // S5g (whole-graph replica groups): graphs longest first (depth, then cell count, then batch
    // index), each to the group whose estimated time after adding it is smallest (ties: lowest group).
    // A group's time: per-level batches of <= 16 cells plus per-cell work: est = Σ_l 2 ceil(n_l/16) + n_l.
    std::vector<int32_t> graph_group;
    if (plan.by_graph) {
        const int32_t NG = b.n_graphs;
        std::vector<std::vector<int32_t>> hist(NG, std::vector<int32_t>(L + 1, 0));
        std::vector<int32_t> depth(NG, 0), cells(NG, 0);
        for (int64_t i = 0; i < N; ++i)
            if (nodes[i].kind != K_HEAD) {
                ++hist[nodes[i].graph][level[i]];
                ++cells[nodes[i].graph];
                depth[nodes[i].graph] = std::max(depth[nodes[i].graph], level[i]);
            }
        std::vector<int32_t> order(NG);
        for (int32_t gi = 0; gi < NG; ++gi) order[gi] = gi;
        std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t c) {
            if (depth[a] != depth[c]) return depth[a] > depth[c];
            return cells[a] > cells[c];
        });
        std::vector<std::vector<int32_t>> gh(G, std::vector<int32_t>(L + 1, 0));
        constexpr int64_t kBatch = 2;   // per-batch overhead in units of one cell (measured sweep)
        auto est_with = [&](int32_t g, int32_t gi) {
            int64_t t = 0;
            for (int32_t l = 0; l <= L; ++l) {
                const int64_t x = gh[g][l] + hist[gi][l];
                t += kBatch * ((x + 15) / 16) + x;
            }
            return t;
        };
        graph_group.resize(NG);
        for (int32_t gi : order) {
            int32_t best = 0;
            int64_t best_t = est_with(0, gi);
            for (int32_t g = 1; g < G; ++g) {
                const int64_t t = est_with(g, gi);
                if (t < best_t) { best = g; best_t = t; }
            }
            for (int32_t l = 0; l <= L; ++l) gh[best][l] += hist[gi][l];
            graph_group[gi] = best;
        }
    }
    for (int32_t p = 0; p < P && !plan.skip_words; ++p) {
        const bool fwd = p <= L;
        const int32_t lv = fwd ? p : 2 * L + 1 - p;
        for (int32_t g = 0; g < G; ++g) { body[g].clear(); load[g] = 0; }
        for (int64_t i : at_level[lv]) {
            int32_t best = 0;
            if (plan.by_graph) {
                best = graph_group[nodes[i].graph];
            } else {
                for (int32_t g = 1; g < G; ++g)
                    if (load[g] < load[best]) best = g;
                load[best] += macs(i);
            }
            emit(body[best], i, fwd);
        }
        int32_t active_prev = 0;
        for (int32_t g = 0; g < G; ++g) active_prev += was_active[g];
        if (p >= 1) targets[p] = (uint32_t)(plan.n_act * active_prev);
        for (int32_t g = 0; g < G; ++g) {
            const bool active = !body[g].empty();
            if (active) {
                if (p >= 1) streams[g].push_back(preamble(OP_W, p));
                streams[g].insert(streams[g].end(), body[g].begin(), body[g].end());
                if (p < P - 1) streams[g].push_back(preamble(OP_S, p + 1));
            }
            was_active[g] = active;
        }
    }

    PHASE(4);
    // ---- header: [G, n_bar, prefix sums], streams, barrier targets (L169) ---------------------
    Script& s = *out;
    s.words.clear();
    if (!plan.skip_words) {
        s.words.push_back((uint32_t)G);
        s.words.push_back((uint32_t)n_bar);
        uint32_t run = 0;
        s.words.push_back(0);
        for (int32_t g = 0; g < G; ++g) { run += (uint32_t)streams[g].size(); s.words.push_back(run); }
        for (int32_t g = 0; g < G; ++g) s.words.insert(s.words.end(), streams[g].begin(), streams[g].end());
        s.words.insert(s.words.end(), targets.begin(), targets.end());
    }
    s.pool_words = cursor;
    s.zero_words = zero_words;
    s.loss_word = loss_word;
    s.n_bar = n_bar;
    s.n_levels = L + 1;
    s.n_nodes = N;
    s.n_heads = 0;
    s.max_token = -1;
    for (const Node& n : nodes) {
        s.n_heads += n.kind == K_HEAD;
        s.max_token = std::max<int64_t>(s.max_token, n.token);
    }
    s.flops = flops;
    s.act_bytes = abytes;
    // replica-group kernel of the binary whole-graph paths: per internal cell the recurrent matvec and
    // its transpose (2 x 8 H^2 MACs), per head the logits, dW_out and dh (3 C H MACs); leaves and dW are
    // GEMMs outside it
    s.kernel_flops = 0.0;
    for (const Node& n : nodes) {
        if (n.kind == K_INT) s.kernel_flops += 2.0 * 16.0 * (double)H * (double)H;
        else if (n.kind == K_HEAD) s.kernel_flops += 2.0 * 3.0 * (double)C * (double)H;
    }
    // device blob: the words, then the operand lists of the per-matrix gradient GEMM (binary cells)
    // (grouped by replica group when graphs are assigned whole, S5g: the GEMM tiles of a group can then
    // start as soon as that group's cluster has finished)
    s.blob = s.words;
    s.lists_off = (int64_t)s.blob.size();
    s.n_int = s.n_leaf = 0;
    const int32_t n_grp = plan.by_graph ? G : 1;
    auto group_of = [&](int64_t i) { return plan.by_graph ? graph_group[nodes[i].graph] : 0; };
    s.int_off.assign(n_grp + 1, 0);
    s.leaf_off.assign(n_grp + 1, 0);
    s.grp_nodes.assign(n_grp, 0);
    s.grp_levels.assign(n_grp, 0);
    for (int64_t i = 0; i < N; ++i) {
        if (nodes[i].kind == K_HEAD) continue;
        const int32_t g = group_of(i);
        ++s.grp_nodes[g];
        s.grp_levels[g] = std::max(s.grp_levels[g], level[i]);
    }
    for (int32_t g = 0; g < n_grp; ++g) {
        s.int_off[g] = (int32_t)s.n_int;
        for (int64_t i = 0; i < N; ++i)
            if (nodes[i].kind == K_INT && group_of(i) == g) {
                const int32_t* ch = kids.data() + nodes[i].ch_begin;
                s.blob.insert(s.blob.end(), {rec[i], rec[ch[0]], rec[ch[1]]});
                ++s.n_int;
            }
    }
    s.int_off[n_grp] = (int32_t)s.n_int;
    for (int32_t g = 0; g < n_grp; ++g) {
        s.leaf_off[g] = (int32_t)s.n_leaf;
        for (int64_t i = 0; i < N; ++i)
            if (nodes[i].kind == K_LEAF && group_of(i) == g) {
                s.blob.insert(s.blob.end(), {rec[i], (uint32_t)nodes[i].token});
                ++s.n_leaf;
            }
    }
    s.leaf_off[n_grp] = (int32_t)s.n_leaf;

    PHASE(5);
    // ---- level-synchronous lowering of the binary cell (Plan::level): per-level node lists ------
    s.lv_int = s.lv_leaf = s.lv_head = -1;
    s.lv_n_int = s.lv_n_leaf = s.lv_n_head = 0;
    s.lv_start.clear();
    if (plan.level && (plan.cell == CELL_BINARY || plan.cell == CELL_RVNN || plan.cell == CELL_TDRNN ||
                       plan.cell == CELL_TDLSTM)) {
        s.lv_int = (int64_t)s.blob.size();
        s.lv_start.assign(L + 2, 0);
        for (int32_t lv = 1; lv <= L + 1; ++lv) {
            s.lv_start[lv] = (int32_t)s.lv_n_int;
            if (lv > L) break;
            for (int64_t i : at_level[lv]) {
                if (nodes[i].kind != K_INT) continue;
                const int32_t* ch = kids.data() + nodes[i].ch_begin;
                s.blob.insert(s.blob.end(), {rec[i], rec[ch[0]], rec[ch[1]], adj[i], adj[ch[0]], adj[ch[1]]});
                ++s.lv_n_int;
            }
        }
        s.lv_leaf = (int64_t)s.blob.size();
        for (int64_t i = 0; i < N; ++i)
            if (nodes[i].kind == K_LEAF) {
                s.blob.insert(s.blob.end(), {rec[i], adj[i], (uint32_t)nodes[i].token});
                ++s.lv_n_leaf;
            }
        s.lv_head = (int64_t)s.blob.size();
        for (int64_t i = 0; i < N; ++i)
            if (nodes[i].kind == K_HEAD) {
                const int32_t* ch = kids.data() + nodes[i].ch_begin;
                s.blob.insert(s.blob.end(), {rec[i], rec[ch[0]], adj[ch[0]], (uint32_t)nodes[i].label});
                ++s.lv_n_head;
            }
    }

    PHASE(6);
    // ---- dataflow lowering of the binary cell for whole-graph groups (vpps_df) ------------------
    // Per group: batches of <= 16 nodes of one opcode, forward levels 1..L then backward levels L..0
    // (level 0 leaves run as a GEMM before the kernel).  Cross-CTA values live in epoch-tagged 64-bit
    // slots so consumers wait on the data itself: HX (h of an internal node with a consumer, 256
    // slots), PART (transposed-product partials of an internal node, [consumer CTA][producer CTA][32]:
    // 16 units of dh_l then 16 of dh_r), HD (head contribution to a labelled node's dh, 256 slots).
    s.df_off = -1;
    s.n_hx = s.n_part = s.n_hd = 0;
    s.df_words = 0;
    if (plan.by_graph && plan.cell == CELL_BINARY) {
        std::vector<int64_t> parent(N, -1), head_of(N, -1);
        std::vector<int32_t> side(N, 0);
        for (int64_t i = 0; i < N; ++i) {
            const int32_t* ch = kids.data() + nodes[i].ch_begin;
            if (nodes[i].kind == K_INT) {
                parent[ch[0]] = i; side[ch[0]] = 0;
                parent[ch[1]] = i; side[ch[1]] = 1;
            } else if (nodes[i].kind == K_HEAD) {
                head_of[ch[0]] = i;
            }
        }
        std::vector<uint32_t> hx(N, NONE), pp(N, NONE), hd(N, NONE);
        for (int64_t i = 0; i < N; ++i) {
            if (nodes[i].kind == K_INT && (parent[i] >= 0 || head_of[i] >= 0)) hx[i] = (uint32_t)s.n_hx++;
            if (nodes[i].kind == K_INT) pp[i] = (uint32_t)s.n_part++;
            if (head_of[i] >= 0) hd[i] = (uint32_t)s.n_hd++;
        }
        auto dsrc = [&](int64_t i) -> uint32_t {
            return parent[i] >= 0 ? (pp[parent[i]] << 1) | (uint32_t)side[i] : NONE;
        };
        std::vector<std::vector<uint32_t>> prog(G);
        auto emit_batches = [&](int32_t g, uint32_t op, const std::vector<int64_t>& list) {
            const size_t cap = op == OP_LEAF_B ? 64 : 16;   // leaf backward needs no shared staging
            for (size_t b0 = 0; b0 < list.size(); b0 += cap) {
                const size_t nb = std::min<size_t>(cap, list.size() - b0);
                std::vector<uint32_t>& w = prog[g];
                w.push_back(op | (uint32_t)(nb << 8));
                for (size_t k = b0; k < b0 + nb; ++k) {
                    const int64_t i = list[k];
                    const int32_t* ch = kids.data() + nodes[i].ch_begin;
                    switch (op) {
                        case OP_INT_F:
                            w.insert(w.end(), {rec[i], hx[i], rec[ch[0]], hx[ch[0]], rec[ch[1]], hx[ch[1]]});
                            break;
                        case OP_HEAD_FB:
                            w.insert(w.end(), {rec[i], rec[ch[0]], (uint32_t)nodes[i].label, hx[ch[0]], hd[ch[0]]});
                            break;
                        case OP_INT_B:
                            w.insert(w.end(), {rec[i], adj[i], dsrc(i), hd[i], pp[i], rec[ch[0]], adj[ch[0]],
                                               rec[ch[1]], adj[ch[1]]});
                            break;
                        default:   // OP_LEAF_B
                            w.insert(w.end(), {rec[i], adj[i], dsrc(i), hd[i]});
                    }
                }
            }
        };
        std::vector<std::vector<int64_t>> lists(5);
        for (int32_t g = 0; g < G; ++g) {
            for (int32_t lv = 1; lv <= L; ++lv) {
                for (auto& l : lists) l.clear();
                for (int64_t i : at_level[lv]) {
                    if (graph_group[nodes[i].graph] != g) continue;
                    if (nodes[i].kind == K_INT) lists[0].push_back(i);
                    else if (nodes[i].kind == K_HEAD) lists[1].push_back(i);
                }
                emit_batches(g, OP_INT_F, lists[0]);
                emit_batches(g, OP_HEAD_FB, lists[1]);   // head forward + backward (dz needs only p)
            }
            for (int32_t lv = L; lv >= 0; --lv) {
                for (auto& l : lists) l.clear();
                for (int64_t i : at_level[lv]) {
                    if (graph_group[nodes[i].graph] != g) continue;
                    if (nodes[i].kind == K_INT) lists[3].push_back(i);
                    else if (nodes[i].kind == K_LEAF) lists[4].push_back(i);
                }
                emit_batches(g, OP_INT_B, lists[3]);
                emit_batches(g, OP_LEAF_B, lists[4]);
            }
        }
        s.df_off = (int64_t)s.blob.size();
        s.blob.push_back((uint32_t)G);
        uint32_t run2 = 0;
        s.blob.push_back(0);
        for (int32_t g = 0; g < G; ++g) { run2 += (uint32_t)prog[g].size(); s.blob.push_back(run2); }
        for (int32_t g = 0; g < G; ++g) s.blob.insert(s.blob.end(), prog[g].begin(), prog[g].end());
        // tagged regions behind the SPEC pool (64-bit slots = 2 words each)
        int64_t cur = align32(s.pool_words);
        // HX: H slots per node; PART: 16 consumer x 16 producer CTAs x 2 (H / 16) slots per parent; HD: H
        s.df_hx = cur;   cur = align32(cur + 2 * H * s.n_hx);
        s.df_part = cur; cur = align32(cur + 2 * 32 * H * s.n_part);
        s.df_hd = cur;   cur = align32(cur + 2 * H * s.n_hd);
        s.df_words = cur - s.pool_words;
    }
    PHASE(7);
    return 0;
}

}  // namespace vpps
