// Weight-matrix distribution over the register files of all CTAs.
//
// SPEC_SCRIPT.md §P.  PAPER.md §III-A1 (L92-115): weight matrices are cut into pieces of whole rows
// (one warp per row, L94) and dealt round-robin over equally sized register partitions of every CTA
// (L92, Fig.4 L88, fn2 L96); partition size Eq.(1); register budget fn6 L127; gradient
// partitions "in the same fashion" L104; one or two CTAs per SM from the aggregate size L106/L241.
#include <algorithm>
#include "host.h"

namespace vpps {

int32_t regs_per_row(int32_t row_max) { return (row_max + 31) / 32; }   // ceil(row_max/warpSize), Eq.(1)

// fn6 (L127): 255 - 31 (interpreter) - 32 (vector cache) = 192 at one 256-thread CTA per SM.
int32_t reg_budget(int32_t tb, int32_t cps) { return std::min(255, 65536 / (tb * cps)) - 63; }

void paper_deal(const std::vector<Shape>& mats, int32_t n_cta, int32_t tb, int32_t rpw, bool pack_rows,
                bool grads, std::vector<DealRow>* rows, int64_t* n_slots) {
    int32_t row_max = 0;
    for (const Shape& s : mats) row_max = std::max(row_max, s.cols);
    const int32_t R = regs_per_row(row_max);
    const int32_t warps = tb / 32;
    struct Piece { int32_t m, first, count, q; };
    std::vector<Piece> pieces;
    for (int32_t m = 0; m < (int32_t)mats.size(); ++m) {
        // rows per warp: rpw, or rpw * floor(R / ceil(c/32)) short rows packed into one slot (R-8)
        const int32_t q = pack_rows ? rpw * (R / regs_per_row(mats[m].cols)) : rpw;
        const int32_t per_piece = warps * q;
        for (int32_t first = 0; first < mats[m].rows; first += per_piece)
            pieces.push_back({m, first, std::min(per_piece, mats[m].rows - first), q});
    }
    int64_t slot = 0;
    if (rows) rows->clear();
    for (int32_t pass = 0; pass < (grads ? 2 : 1); ++pass) {
        if (pass == 1) slot = (slot + n_cta - 1) / n_cta * n_cta;   // dW restarts on a slot boundary
        for (const Piece& p : pieces) {
            const int32_t cta = (int32_t)(slot % n_cta), part = (int32_t)(slot / n_cta);
            if (rows)
                for (int32_t k = 0; k < p.count; ++k)
                    rows->push_back({p.m, p.first + k, cta, part, k / p.q, pass});
            ++slot;
        }
    }
    *n_slots = slot;
}

int32_t paper_choose_cps(const std::vector<Shape>& mats, int32_t n_sm, int32_t tb, int32_t rpw, bool pack_rows) {
    int32_t row_max = 0;
    for (const Shape& s : mats) row_max = std::max(row_max, s.cols);
    const int32_t R = regs_per_row(row_max);
    const int32_t n_cta = 2 * n_sm;
    int64_t slots = 0;
    paper_deal(mats, n_cta, tb, rpw, pack_rows, true, nullptr, &slots);
    const int64_t per_cta = (slots + n_cta - 1) / n_cta;
    return per_cta <= reg_budget(tb, 2) / (rpw * R) ? 2 : 1;
}

// SPEC P1: atoms 0..H-1 are gate-colocated unit bundles, atom H the head; atom a -> CTA a mod n_g,
// slot a / n_g of every replica group.
bool unit_plan(int32_t cell, int32_t H, int32_t E, int32_t C, int32_t n_sm, int32_t cps, int32_t G,
               Plan* out, std::string* err) {
    Plan& p = *out;
    p.cell = cell; p.H = H; p.E = E; p.C = C; p.G = G;
    p.n_cta = n_sm * cps;
    if (G < 1 || p.n_cta % G != 0) { *err = "groups must divide the CTA count"; return false; }
    p.n_g = p.n_cta / G;
    p.n_act = std::min(p.n_g, H + 1);
    const int32_t need = (H + p.n_g - 1) / p.n_g;
    p.umax = 1;
    while (p.umax < need) p.umax *= 2;
    if (p.umax > 16) { *err = "NOFIT: more than 16 hidden units per CTA"; return false; }

    // (matrix, gate rows of unit j) for each cell family, matrices in parameter order
    struct Block { int32_t matrix, gates, cols; };
    std::vector<Block> blocks;
    int32_t head_matrix = 0;
    switch (cell) {
        case CELL_LSTM: blocks = {{0, 4, E}, {1, 4, H}}; head_matrix = 2; break;
        case CELL_BINARY: blocks = {{0, 3, E}, {1, 3, 2 * H}, {2, 1, H}, {3, 1, H}}; head_matrix = 4; break;
        case CELL_CHILDSUM: blocks = {{0, 3, E}, {1, 1, E}, {2, 3, H}, {3, 1, H}}; head_matrix = 4; break;
        default: *err = "unknown cell"; return false;
    }
    p.table.clear();
    for (int32_t g = 0; g < G; ++g) {
        for (int32_t a = 0; a <= H; ++a) {
            const int32_t cta = g * p.n_g + a % p.n_g, slot = a / p.n_g;
            auto emit = [&](int32_t m, int32_t r, int32_t c, int32_t st) {
                const int32_t row8[8] = {m, r, c, g, cta, slot, st, st};
                p.table.insert(p.table.end(), row8, row8 + 8);
            };
            if (a < H) {
                for (const Block& b : blocks)
                    for (int32_t k = 0; k < b.gates; ++k) emit(b.matrix, k * H + a, b.cols, 0);
            } else {
                for (int32_t r = 0; r < C; ++r) emit(head_matrix, r, H, 1);
            }
        }
    }
    return true;
}

}  // namespace vpps
