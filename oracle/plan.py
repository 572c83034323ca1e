"""Weight-matrix distribution (TEST INFRASTRUCTURE ONLY — see oracle/__init__.py).

Written from SPEC_SCRIPT.md §P, step by step, in the paper's terms:
  paper_deal()   — P0: round-robin of row pieces over register partitions of all CTAs
                   (§III-A1, Fig.4 L88, L94, fn2 L96, Eq.(1), fn6 L127,
                   gradient partitions L104, CTAs/SM L106/L241)
  unit_plan()    — P1: the B200 plan; the same round-robin applied to gate-colocated unit bundles
"""
from __future__ import annotations

import math

WARP = 32


def regs_per_row(row_max: int) -> int:
    """R = ceil(row_max / warpSize) (Eq.(1))."""
    return -(-row_max // WARP)


def partition_size(tb: int, rpw: int, row_max: int) -> int:
    """P_size = TBSize * rpw * ceil(row_max / warpSize) (Eq.(1))."""
    return tb * rpw * regs_per_row(row_max)


def reg_budget(tb: int, cps: int) -> int:
    """Registers per thread left for weights: 255 - 31 (interpreter) - 32 (vector cache) at one
    256-wide CTA per SM (fn6, L127); min(255, 65536/(TB*cps)) - 63 in general (reading R-11)."""
    return min(255, 65536 // (tb * cps)) - 63


def rpw_max(tb: int, cps: int, row_max: int) -> int:
    return reg_budget(tb, cps) // regs_per_row(row_max)


def rows_per_warp(c: int, rpw: int, R: int, pack_rows: bool) -> int:
    """q_m (SPEC P0.2, reading R-8)."""
    return rpw * (R // regs_per_row(c)) if pack_rows else rpw


def paper_deal(shapes, n_cta: int, tb: int, rpw: int, pack_rows: bool = True, grads: bool = False):
    """P0.3-P0.5.  Returns (rows, n_slots) where rows is a list of
    (matrix, row, cta, partition, warp, is_grad) and n_slots the number of slots used."""
    R = regs_per_row(max(c for (_, c) in shapes))
    nw = tb // WARP
    pieces = []                                  # (matrix, first row, n rows, q)
    for m, (r, c) in enumerate(shapes):
        q = rows_per_warp(c, rpw, R, pack_rows)
        per = nw * q
        for r0 in range(0, r, per):
            pieces.append((m, r0, min(per, r - r0), q))
    out = []
    s = 0
    for is_grad in ([0, 1] if grads else [0]):
        if is_grad:
            s = -(-s // n_cta) * n_cta           # P0.5: round up to a multiple of n_cta
        for (m, r0, n, q) in pieces:
            cta, part = s % n_cta, s // n_cta
            for k in range(n):
                out.append((m, r0 + k, cta, part, k // q, is_grad))
            s += 1
    return out, s


def fits_in_registers(shapes, n_sm: int, cps: int, tb: int = 256, rpw: int = 1, pack_rows: bool = True) -> bool:
    R = regs_per_row(max(c for (_, c) in shapes))
    n_cta = n_sm * cps
    _, n_slots = paper_deal(shapes, n_cta, tb, rpw, pack_rows, grads=True)
    parts_per_cta = -(-n_slots // n_cta)
    return parts_per_cta <= reg_budget(tb, cps) // (rpw * R)


def choose_cps(shapes, n_sm: int, tb: int = 256, rpw: int = 1, pack_rows: bool = True) -> int:
    """P0.7: two CTAs per SM iff everything fits in registers at two, else one (L106, L241)."""
    return 2 if fits_in_registers(shapes, n_sm, 2, tb, rpw, pack_rows) else 1


# ------------------------------------------------------------------------------------------
# P1: B200 unit-bundle plan
# ------------------------------------------------------------------------------------------
def unit_rows(cell: str, H: int, j: int):
    """(matrix index, row) pairs of the gate-colocated bundle of hidden unit j (SPEC P1.6)."""
    if cell == "lstm":        # W, U, W_out, b, b_out
        return [(0, g * H + j) for g in range(4)] + [(1, g * H + j) for g in range(4)]
    if cell == "binary":      # W_iou, U_iou, U_fl, U_fr, W_out, ...
        return [(0, g * H + j) for g in range(3)] + [(1, g * H + j) for g in range(3)] + [(2, j), (3, j)]
    if cell == "childsum":    # W_iou, W_f, U_iou, U_f, W_out, ...
        return ([(0, g * H + j) for g in range(3)] + [(1, j)] + [(2, g * H + j) for g in range(3)] + [(3, j)])
    raise ValueError(cell)


HEAD_MATRIX = {"lstm": 2, "binary": 4, "childsum": 4}


def unit_plan(cell: str, H: int, E: int, C: int, n_sm: int, cps: int = 1, G: int = 1):
    """Returns dict(n_cta, n_g, n_act, umax, table) with table rows
    (matrix, row, cols, group, cta, slot, storage, grad_storage)."""
    n_cta = n_sm * cps
    if G < 1 or n_cta % G:
        raise ValueError("G must divide n_cta")
    n_g = n_cta // G
    umax_needed = -(-H // n_g)
    umax = 1
    while umax < umax_needed:
        umax *= 2
    if umax > 16:
        raise ValueError("NOFIT: more than 16 units per CTA")
    cols = {
        "lstm": [E, H, H], "binary": [E, 2 * H, H, H, H], "childsum": [E, E, H, H, H],
    }[cell]
    table = []
    for g in range(G):
        for a in range(H + 1):
            cta = g * n_g + (a % n_g)
            slot = a // n_g
            if a < H:
                for (m, r) in unit_rows(cell, H, a):
                    table.append((m, r, cols[m], g, cta, slot, 0, 0))
            else:
                m = HEAD_MATRIX[cell]
                for r in range(C):
                    table.append((m, r, cols[m], g, cta, slot, 1, 1))
    return dict(n_cta=n_cta, n_g=n_g, n_act=min(n_g, H + 1), umax=umax, table=table)
