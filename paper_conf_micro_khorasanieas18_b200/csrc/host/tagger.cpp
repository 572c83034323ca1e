// Batch lowering of LSTM chains for the level-synchronous path: the BiLSTM tagger (M2; PAPER L265, L281:
// the NER tagger of Table III) and the LSTM LM with a large vocabulary (config 3): sentences are concatenated into T positions; time step t of the forward LSTM
// runs position t of every sentence longer than t, step t of the backward LSTM position len-1-t (the
// paper's level sort, L139, of the two chains).  The loss is the sum over labelled positions (L205).
#include <algorithm>
#include "host.h"

namespace vpps {

int build_tagger_script(const Plan& plan, const BatchIn& b, int64_t n_input_rows, Script* out, std::string* err) {
    if (b.n_graphs < 0 || (b.n_graphs > 0 && (!b.graph_ptr || !b.child_ptr || !b.token || !b.label))) {
        *err = "null batch array";
        return -1;
    }
    Script& s = *out;
    s = Script{};
    std::vector<int32_t> off(b.n_graphs + 1, 0), len(b.n_graphs, 0);
    for (int32_t g = 0; g < b.n_graphs; ++g) {
        const int32_t first = b.graph_ptr[g], last = b.graph_ptr[g + 1];
        if (last < first) { *err = "graph_ptr not monotone"; return -4; }
        for (int32_t v = first; v < last; ++v) {
            const int32_t t = v - first, c0 = b.child_ptr[v], c1 = b.child_ptr[v + 1];
            const bool ok = (t == 0 && c1 == c0) || (t > 0 && c1 == c0 + 1 && b.children[c0] == t - 1);
            if (!ok) { *err = "chain: node t has the single child t-1"; return -4; }
            const bool rare = plan.cell == CELL_BILSTM_CHAR && b.char_ptr && b.char_ptr[v + 1] > b.char_ptr[v];
            if (!rare && (b.token[v] < 0 || b.token[v] >= n_input_rows)) { *err = "token out of range"; return -4; }
            if (plan.cell != CELL_BILSTM_CHAR && b.char_ptr && b.char_ptr[v + 1] > b.char_ptr[v]) {
                *err = "character spellings need the BiLSTMwChar cell";
                return -4;
            }
            if (b.label[v] < -1 || b.label[v] >= plan.C) { *err = "label out of range"; return -4; }
            if (!rare) s.max_token = std::max<int64_t>(s.max_token, b.token[v]);
            s.n_heads += b.label[v] >= 0;
        }
        len[g] = last - first;
        off[g + 1] = off[g] + len[g];
    }
    const int32_t T = off[b.n_graphs];
    const int32_t maxlen = b.n_graphs ? *std::max_element(len.begin(), len.end()) : 0;
    s.tg_T = T;
    s.n_nodes = T;
    s.n_levels = maxlen;
    auto is_rare = [&](int32_t v) {
        return plan.cell == CELL_BILSTM_CHAR && b.char_ptr && b.char_ptr[v + 1] > b.char_ptr[v];
    };
    s.tg_tok = (int64_t)s.blob.size();
    for (int32_t g = 0; g < b.n_graphs; ++g)
        for (int32_t t = 0; t < len[g]; ++t) {
            const int32_t v = b.graph_ptr[g] + t;
            s.blob.push_back(is_rare(v) ? NONE : (uint32_t)b.token[v]);   // rare words: no table row
        }
    s.tg_lab = (int64_t)s.blob.size();
    for (int32_t g = 0; g < b.n_graphs; ++g)
        for (int32_t t = 0; t < len[g]; ++t) s.blob.push_back((uint32_t)b.label[b.graph_ptr[g] + t]);
    // step lists with the sentences longest first: the sentences still running at step t are then a prefix
    // of those at step t-1, so row r of step t continues row r of step t-1 (the device reads h_prev and the
    // successor's dh as row-aligned step blocks, without gathers or scatters)
    std::vector<int32_t> order(b.n_graphs);
    for (int32_t g = 0; g < b.n_graphs; ++g) order[g] = g;
    std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t c) { return len[a] > len[c]; });
    s.tg_start.assign(maxlen + 1, 0);
    s.tg_fpos = (int64_t)s.blob.size();
    int32_t k = 0;
    for (int32_t t = 0; t < maxlen; ++t) {
        s.tg_start[t] = k;
        for (int32_t g : order)
            if (len[g] > t) { s.blob.push_back((uint32_t)(off[g] + t)); ++k; }
    }
    s.tg_start[maxlen] = k;
    s.tg_bpos = (int64_t)s.blob.size();
    for (int32_t t = 0; t < maxlen; ++t)
        for (int32_t g : order)
            if (len[g] > t) s.blob.push_back((uint32_t)(off[g] + len[g] - 1 - t));
    double char_flops = 0.0;
    if (plan.cell == CELL_BILSTM_CHAR) {
        // plus the character BiLSTM (Hc = E / 2 per direction over Ec-wide character embeddings): per
        // character and direction the input and (after the first character) recurrent products
        const double Hc = plan.E / 2, Ec = plan.ec;
        int64_t tc = 0, rw = 0;
        for (int32_t v = 0; v < (b.n_graphs ? b.graph_ptr[b.n_graphs] : 0); ++v)
            if (is_rare(v)) { tc += b.char_ptr[v + 1] - b.char_ptr[v]; ++rw; }
        char_flops = 2.0 * ((double)tc * 24.0 * Hc * Ec + (double)(tc - rw) * 24.0 * Hc * Hc);
    }
    // sentence table of the register-resident recurrence (SPEC §L; vpps_chain.cu): sentences longest first,
    // each to the group (per direction) with the smallest total length so far (ties: lowest group), at most
    // 64 per group; [G, pre_0 .. pre_G, (off, len) per sentence], direction 1's groups repeat direction 0's
    s.tg_chain = -1;
    if (plan.chain_g > 0 && T > 0) {
        const int32_t Gd = plan.chain_g, dirs = plan.cell == CELL_BILSTM || plan.cell == CELL_BILSTM_CHAR ? 2 : 1;
        std::vector<std::vector<int32_t>> mem(Gd);
        std::vector<int64_t> load(Gd, 0);
        bool fits = true;
        for (int32_t g : order) {
            if (len[g] == 0) continue;
            int32_t best = -1;
            for (int32_t q = 0; q < Gd; ++q)
                if ((int32_t)mem[q].size() < 64 && (best < 0 || load[q] < load[best])) best = q;
            if (best < 0) { fits = false; break; }
            mem[best].push_back(g);
            load[best] += len[g];
        }
        if (fits) {
            s.tg_chain = (int64_t)s.blob.size();
            const int32_t G = Gd * dirs;
            s.blob.push_back((uint32_t)G);
            uint32_t run = 0;
            s.blob.push_back(0);
            for (int32_t q = 0; q < G; ++q) { run += (uint32_t)mem[q % Gd].size(); s.blob.push_back(run); }
            for (int32_t q = 0; q < G; ++q)
                for (int32_t g : mem[q % Gd]) { s.blob.push_back((uint32_t)off[g]); s.blob.push_back((uint32_t)len[g]); }
        }
    }
    // BiLSTMwChar: the spellings of the rare positions, concatenated in position order, and their chain table
    if (plan.cell == CELL_BILSTM_CHAR) {
        std::vector<uint32_t> ctok, cword, rare(T, NONE), rlist;
        int32_t R = 0;
        for (int32_t g = 0; g < b.n_graphs; ++g)
            for (int32_t t = 0; t < len[g]; ++t) {
                const int32_t v = b.graph_ptr[g] + t;
                if (!is_rare(v)) continue;
                const int32_t c0 = b.char_ptr[v], c1 = b.char_ptr[v + 1];
                rlist.insert(rlist.end(), {(uint32_t)(off[g] + t), (uint32_t)ctok.size(), (uint32_t)(c1 - c0)});
                for (int32_t k = c0; k < c1; ++k) {
                    if (b.chars[k] < 0 || b.chars[k] >= plan.vc) { *err = "character id out of range"; return -4; }
                    ctok.push_back((uint32_t)b.chars[k]);
                    cword.push_back((uint32_t)R);
                }
                rare[off[g] + t] = (uint32_t)R++;
            }
        s.tc_T = (int64_t)ctok.size();
        s.tc_R = R;
        s.tc_tok = (int64_t)s.blob.size(); s.blob.insert(s.blob.end(), ctok.begin(), ctok.end());
        s.tc_word = (int64_t)s.blob.size(); s.blob.insert(s.blob.end(), cword.begin(), cword.end());
        s.tc_rare = (int64_t)s.blob.size(); s.blob.insert(s.blob.end(), rare.begin(), rare.end());
        s.tc_list = (int64_t)s.blob.size(); s.blob.insert(s.blob.end(), rlist.begin(), rlist.end());
        // character chains: the same table rule as the words (SPEC §L), over the spellings, two directions
        s.tc_chain = -1;
        if (R > 0 && plan.chain_gc > 0) {
            const int32_t Gd = plan.chain_gc;
            std::vector<int32_t> ro(R);
            for (int32_t r = 0; r < R; ++r) ro[r] = r;
            std::stable_sort(ro.begin(), ro.end(), [&](int32_t a, int32_t c) { return rlist[3 * a + 2] > rlist[3 * c + 2]; });
            std::vector<std::vector<int32_t>> mem(Gd);
            std::vector<int64_t> load(Gd, 0);
            bool fits = true;
            for (int32_t r : ro) {
                int32_t best = -1;
                for (int32_t q = 0; q < Gd; ++q)
                    if ((int32_t)mem[q].size() < 64 && (best < 0 || load[q] < load[best])) best = q;
                if (best < 0) { fits = false; break; }
                mem[best].push_back(r);
                load[best] += rlist[3 * r + 2];
            }
            if (!fits) { *err = "too many rare words for the character recurrence's groups"; return -1; }
            s.tc_chain = (int64_t)s.blob.size();
            const int32_t G = 2 * Gd;
            s.blob.push_back((uint32_t)G);
            uint32_t run = 0;
            s.blob.push_back(0);
            for (int32_t q = 0; q < G; ++q) { run += (uint32_t)mem[q % Gd].size(); s.blob.push_back(run); }
            for (int32_t q = 0; q < G; ++q)
                for (int32_t r : mem[q % Gd]) { s.blob.push_back(rlist[3 * r + 1]); s.blob.push_back(rlist[3 * r + 2]); }
        }
    }
    // pool: the loss word only (the tagger's activations live in the path's work buffers)
    s.loss_word = 0;
    s.zero_words = 32;
    s.pool_words = 32;
    // algorithmic FLOPs (oracle.models.flop_count): per position and direction the input
    // product W x (fwd, dW, dx: 3 x 2 FLOP per MAC), after a direction's first step the recurrent product
    // U h; per labelled position the MLP (2H x M) and the tag head (M x C) of the tagger, the head (H x C)
    // of the LM / GRU
    int32_t S = 0;
    for (int32_t g = 0; g < b.n_graphs; ++g) S += len[g] > 0;
    const double H = plan.H, E = plan.E, C = plan.C, M = plan.mlp;
    const double Tt = T, Tr = (double)T - S;   // positions with a predecessor in a direction
    if (plan.cell == CELL_BILSTM || plan.cell == CELL_BILSTM_CHAR)
        s.flops = 2.0 * (Tt * 24.0 * H * E + Tr * 24.0 * H * H) + (double)s.n_heads * (12.0 * H * M + 6.0 * M * C);
    else if (plan.cell == CELL_GRU)   // GRU chains: 3 gates, one direction, head on h
        s.flops = Tt * 18.0 * H * E + Tr * 18.0 * H * H + (double)s.n_heads * 6.0 * C * H;
    else   // LSTM LM: one direction, head on h
        s.flops = Tt * 24.0 * H * E + Tr * 24.0 * H * H + (double)s.n_heads * 6.0 * C * H;
    s.flops += char_flops;
    return 0;
}

}  // namespace vpps
