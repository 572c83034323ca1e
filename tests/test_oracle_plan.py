"""Pins of oracle/plan.py and oracle/script.py against the paper's own worked examples and
numbers (CPU only).  Exact script words beyond these pins are "parity unpinned" by the paper
and are checked bit-exactly against the independent C++ implementation (test_host_parity.py)."""
import numpy as np
import pytest

import synth
from oracle import plan, script
from oracle import models as M


def test_eq1_partition_size_fig4():
    # Fig.4 caption (L88): CTA width 128, partition size 1024 = 8 thread registers per partition,
    # row length 128 and two rows per warp (L94) -> Eq.(1): 128 * 2 * ceil(128/32) = 1024.
    assert plan.partition_size(128, 2, 128) == 1024
    assert plan.partition_size(128, 2, 128) // 128 == 8


def test_fn6_rpw_max():
    # fn6 (L127): 255 - 31 - 32 = 192 registers at one CTA per SM; L115: row_max 1024 -> rpw_max 6
    assert plan.reg_budget(256, 1) == 192
    assert plan.rpw_max(256, 1, 1024) == 6


def test_fig4_row8_of_B_in_warp0_of_cta3():
    # L94: "row 8 with the length 128 in Matrix B is distributed across 128 registers of warp 0 in
    # CTA 3" and "two consecutive rows of matrix B are given to each warp".  4 CTAs, width 128.
    for rows_a in (9, 12, 16, 41):
        rows, _ = plan.paper_deal([(rows_a, 128), (24, 128)], n_cta=4, tb=128, rpw=2)
        where = {(m, r): (cta, part, warp) for (m, r, cta, part, warp, _) in rows}
        cta, part, warp = where[(1, 8)]
        assert (cta, warp) == (3, 0), rows_a
        assert where[(1, 9)][2] == 0 and where[(1, 10)][2] == 1     # two consecutive rows per warp


def _m4_shapes(H, E, C=5):
    return [s for (_, s) in M.param_shapes("binary", H, E, C) if len(s) == 2]


def test_l241_occupancy_titan_v():
    # L241: E = 128 (Fig.9), Titan V (80 SMs, L211): H = 256 -> 25% occupancy (2 CTAs/SM),
    # H = 384 -> 12.5% (1 CTA/SM).  L106: up to two CTAs of width 256 per SM.
    assert plan.choose_cps(_m4_shapes(256, 128), n_sm=80) == 2
    assert plan.choose_cps(_m4_shapes(384, 128), n_sm=80) == 1


def test_unit_plan_tgt():
    p = plan.unit_plan("binary", 256, 256, 5, n_sm=148)
    assert p["umax"] == 2 and p["n_act"] == 148
    seen = {}
    for (m, r, cols, g, cta, slot, st, gst) in p["table"]:
        seen.setdefault((m, r), []).append((cta, slot))
    # every matrix row of the model is placed exactly once (one replica)
    for m, (rr, cc) in enumerate(_m4_shapes(256, 256)):
        for r in range(rr):
            assert len(seen[(m, r)]) == 1
    # unit j's gate rows are colocated on CTA j mod 148 (gate colocation), head on CTA 256 mod 148
    for j in (0, 107, 108, 147, 148, 255):
        cta = j % 148
        for (m, r) in plan.unit_rows("binary", 256, j):
            assert seen[(m, r)] == [(cta, j // 148)]
    assert seen[(4, 0)] == [(256 % 148, 1)]


def test_unit_plan_groups_replicate():
    p = plan.unit_plan("lstm", 32, 32, 16, n_sm=148, G=4)
    assert p["n_g"] == 37 and p["n_act"] == 33 and p["umax"] == 1
    per_group = {}
    for row in p["table"]:
        per_group.setdefault(row[3], []).append((row[0], row[1]))
    assert all(sorted(v) == sorted(per_group[0]) for v in per_group.values())


def _fig6_batch():
    # two trees Z = INT(X = INT(a, b), c) where the inner node X carries a label (head at level 2)
    t = [((), 0, -1), ((), 1, -1), ((0, 1), -1, 1), ((), 2, -1), ((2, 3), -1, -1)]
    return [t, t]


SIZES = {0x10: 4, 0x11: 6, 0x20: 3, 0x21: 4, 0x22: 4, 0x23: 7, 0x40: 4, 0x41: 5}


def parse_stream(st):
    """[(op, len)] of a stream (S/W are one word; CS sizes depend on len)."""
    out, i = [], 0
    while i < len(st):
        op, ln = st[i] & 0xFF, st[i] >> 8
        size = 1 if op in (1, 2) else SIZES.get(op, 3 + ln if op == 0x30 else 4 + 2 * ln)
        out.append((op, ln))
        i += size
    assert i == len(st)
    return out


def test_fig6d_idle_vpp_neither_waits_nor_signals():
    # Fig.6(d) (L149-155): VPP#3 runs "V203, S(1), W(2), v24, S(3)": busy in levels 0 and 2, idle in
    # level 1, it signals barrier 1, skips W(1)/S(2), waits on barrier 2.
    s = script.build("binary", _fig6_batch(), H=4, E=4, C=3, G=4, n_act=5)
    w = s["words"]
    G, nbar = w[0], w[1]
    pre = w[2:2 + G + 1]
    base = 2 + G + 1
    ops = parse_stream(w[base + pre[3]: base + pre[4]])
    S, W = script.OP["S"], script.OP["W"]
    assert ops[:5] == [(script.OP["LEAF_F"], 4), (S, 1), (W, 2), (script.OP["HEAD_F"], 4), (S, 3)]
    assert (W, 1) not in ops and (S, 2) not in ops
    # barrier 2 is signalled by the level-1 participants only (groups 0 and 1), 5 CTAs each
    targets = w[-(nbar + 1):]
    assert targets[2] == 2 * 5 and targets[1] == 4 * 5


def test_sw_rule_and_encoding_sizes():
    rng = np.random.default_rng(3)
    for cell in ("binary", "childsum", "lstm"):
        graphs = synth.tree_batch(rng, 5, (2, 9), 10, 3) if cell != "lstm" else \
            [synth.chain(rng, int(rng.integers(2, 7)), 3) for _ in range(5)]
        for G in (1, 2, 4):
            s = script.build(cell, graphs, H=8, E=4, C=3, G=G, n_act=9)
            w = s["words"]
            assert w[0] == G
            pre = w[2:2 + G + 1]
            base = 2 + G + 1
            assert pre[0] == 0 and base + pre[G] + s["n_bar"] + 1 == len(w)     # L169 header
            for g in range(G):
                st = w[base + pre[g]: base + pre[g + 1]]
                i = 0
                waited, signalled = set(), set()
                while i < len(st):
                    op, ln = st[i] & 0xFF, st[i] >> 8
                    if op in (1, 2):                 # S/W are one 4-byte word (L165)
                        (signalled if op == 1 else waited).add(ln)
                        i += 1
                        continue
                    size = {0x10: 4, 0x11: 6, 0x20: 3, 0x21: 4, 0x22: 4, 0x23: 7, 0x40: 4, 0x41: 5}.get(op)
                    if op == 0x30:
                        size = 3 + ln
                    if op == 0x31:
                        size = 4 + 2 * ln
                    assert size is not None
                    # input tensor length in the preamble (L159)
                    if op in (0x20, 0x21):
                        assert ln == 4
                    if op in (0x22, 0x23):
                        assert ln == 16
                    i += size
                assert i == len(st)
                # every wait is on a barrier some group signals; signals precede the matching wait
                assert waited <= set(range(1, s["n_bar"] + 1))


def test_pool_records_do_not_overlap():
    rng = np.random.default_rng(5)
    graphs = synth.tree_batch(rng, 6, (2, 12), 10, 3)
    s = script.build("binary", graphs, H=8, E=8, C=3)
    spans = []
    for i, n in enumerate(s["nodes"]):
        size = {"LEAF": 40, "INT": 56, "HEAD": 4}[n["kind"]]
        spans.append((s["rec"][i], s["rec"][i] + size))
        if n["kind"] != "HEAD":
            spans.append((s["adj"][i], s["adj"][i] + 16))
            assert s["adj"][i] < s["zero_words"]
        assert s["rec"][i] >= s["zero_words"] and s["rec"][i] % 32 == 0
    spans.sort()
    assert all(a[1] <= b[0] for a, b in zip(spans, spans[1:]))
    assert s["loss_word"] >= s["n_bar"] + 1


def test_device_lowering_invariants():
    """oracle device_lowering (SPEC §D) against what the schedule must guarantee (L139/L141/L167): every
    internal cell is computed once forward (after its children) and once backward (after its parent), every
    leaf once backward, every head once, each group only touches its own graphs, and the slot numbers are
    distinct."""
    import synth
    rng = np.random.default_rng(3)
    for G in (1, 4):
        graphs = synth.tree_batch(rng, 12, (1, 30), 40, 5)
        graphs.append([((), 0, 1), ((), 1, -1), ((0, 1), -1, 3), ((), 2, -1), ((2, 3), -1, 0)])
        ref = script.build("binary", graphs, 16, 16, 5, G=G, n_act=16, by_graph=True)
        low = script.device_lowering(ref)
        w = low["lists"][low["df_off"]:]
        assert w[0] == G
        pre = w[1:G + 2]
        rec_id = {r: i for i, r in enumerate(ref["rec"])}
        seen_f, seen_b, heads, hx_seen, pp_seen = {}, {}, set(), set(), set()
        t = 0
        for g in range(G):
            pos, end = G + 2 + pre[g], G + 2 + pre[g + 1]
            while pos < end:
                op, nb = w[pos] & 0xFF, w[pos] >> 8
                sz = {0x22: 6, 0x42: 5, 0x23: 9, 0x21: 4}[op]
                assert 1 <= nb <= (64 if op == 0x21 else 16)
                for k in range(nb):
                    e = w[pos + 1 + k * sz: pos + 1 + (k + 1) * sz]
                    i = rec_id[e[0]]
                    node = ref["nodes"][i]
                    assert ref["graph_group"][node["graph"]] == g
                    t += 1
                    if op == 0x22:
                        assert i not in seen_f
                        for c in node["children"]:
                            assert ref["nodes"][c]["kind"] == "LEAF" or c in seen_f
                        seen_f[i] = t
                        if e[1] != script.NONE:
                            assert e[1] not in hx_seen
                            hx_seen.add(e[1])
                    elif op == 0x42:
                        assert rec_id[e[1]] == node["children"][0] and (ref["nodes"][rec_id[e[1]]]["kind"] == "LEAF"
                                                                         or rec_id[e[1]] in seen_f)
                        heads.add(i)
                    else:
                        assert i not in seen_b
                        if e[2] != script.NONE:       # dsrc: the parent's PART slot, already backward
                            par = [p for p, n in enumerate(ref["nodes"]) if i in n["children"] and n["kind"] == "INT"]
                            assert par and par[0] in seen_b
                        seen_b[i] = t
                        if op == 0x23:
                            assert e[4] not in pp_seen
                            pp_seen.add(e[4])
                pos += 1 + nb * sz
        n_int = sum(n["kind"] == "INT" for n in ref["nodes"])
        n_leaf = sum(n["kind"] == "LEAF" for n in ref["nodes"])
        n_head = sum(n["kind"] == "HEAD" for n in ref["nodes"])
        assert len(seen_f) == n_int and len(seen_b) == n_int + n_leaf and len(heads) == n_head
        assert len(pp_seen) == n_int == low["n_part"] and len(hx_seen) == low["n_hx"]
