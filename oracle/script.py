"""Script generation (TEST INFRASTRUCTURE ONLY — see oracle/__init__.py).

Written from SPEC_SCRIPT.md §S and §E in the paper's order (§III-B1):
super-graph with summed loss (L205) -> level sort by maximum depth from the sources (L139) ->
forward traversal emitting one CISC instruction per node (L141, L159) -> signal/wait between
consecutive levels (L165) -> reverse traversal for back-propagation (L167) with min-load
assignment (L167) -> per-VPP scripts concatenated behind the prefix sum of their lengths (L169).
"""
from __future__ import annotations

NONE = 0xFFFFFFFF
OP = dict(S=0x01, W=0x02, LSTM_F=0x10, LSTM_B=0x11, LEAF_F=0x20, LEAF_B=0x21, INT_F=0x22, INT_B=0x23,
          CS_F=0x30, CS_B=0x31, HEAD_F=0x40, HEAD_B=0x41)


def _a32(x: int) -> int:
    return (x + 31) // 32 * 32


def pre(op: str, length: int) -> int:
    """4-byte preamble: operation type and input tensor length (L159; reading R-16)."""
    assert 0 <= length < (1 << 24)
    return OP[op] | (length << 8)


def build(cell: str, graphs, H: int, E: int, C: int, G: int = 1, n_act: int = 148, by_graph: bool = False):
    """Returns dict(words, pool_words, zero_words, loss_word, n_bar, levels, nodes).

    by_graph: SPEC S5g — whole graphs are assigned to groups (longest first, smallest estimated group time)
    instead of single nodes per level."""
    # S1/S2: super-graph node list
    nodes = []          # dict(kind, graph, cell(local), children(global ids), token, label, cellnode)
    for b, g in enumerate(graphs):
        base = len(nodes)
        for v, (ch, tok, lab) in enumerate(g):
            if cell == "binary":
                kind = "LEAF" if len(ch) == 0 else "INT"
            elif cell == "childsum":
                kind = "CS"
            else:
                kind = "LSTM"
            nodes.append(dict(kind=kind, children=[base + k for k in ch], token=tok, label=lab, graph=b))
        for v, (ch, tok, lab) in enumerate(g):
            if lab >= 0:
                nodes.append(dict(kind="HEAD", children=[base + v], token=-1, label=lab, graph=b))
    # S3: levels
    level = []
    for n in nodes:
        level.append(0 if not n["children"] else 1 + max(level[k] for k in n["children"]))
    L = max(level)
    # S7: pool plan
    n_bar = 2 * L + 1
    z_loss = _a32(n_bar + 1)
    off = _a32(z_loss + 1)
    adj = [NONE] * len(nodes)
    for i, n in enumerate(nodes):
        if n["kind"] != "HEAD":
            adj[i] = off
            off = _a32(off + 2 * H)
    zero_words = off
    rec = [0] * len(nodes)
    for i, n in enumerate(nodes):
        rec[i] = off
        nch = len(n["children"])
        # forward fields, then the gate gradients written by the backward pass (SPEC §S7)
        size = {"LSTM": (6 + 4) * H, "LEAF": (5 + 3) * H, "INT": (7 + 5) * H, "CS": (5 + nch + 3 + nch) * H,
                "HEAD": C + 1}[n["kind"]]
        off = _a32(off + size)
    pool_words = off

    def cost(n):
        k = n["kind"]
        if k == "LEAF":
            return 3 * H * E
        if k == "INT":
            return 6 * H * H + 2 * H * H
        if k == "CS":
            return (4 * H * E if n["token"] >= 0 else 0) + (3 * H * H + len(n["children"]) * H * H
                                                            if n["children"] else 0)
        if k == "LSTM":
            return 4 * H * E + (4 * H * H if n["children"] else 0)
        return C * H

    def tok(t):
        return NONE if t < 0 else t

    def instr(i, fwd):
        n = nodes[i]
        k = n["kind"]
        ch = n["children"]
        if k == "LEAF":
            return [pre("LEAF_F", E), rec[i], n["token"]] if fwd else [pre("LEAF_B", E), rec[i], adj[i], n["token"]]
        if k == "INT":
            l, r = ch
            return ([pre("INT_F", 2 * H), rec[i], rec[l], rec[r]] if fwd else
                    [pre("INT_B", 2 * H), rec[i], adj[i], rec[l], adj[l], rec[r], adj[r]])
        if k == "LSTM":
            p = ch[0] if ch else None
            if fwd:
                return [pre("LSTM_F", E + H), rec[i], n["token"], rec[p] if p is not None else NONE]
            return [pre("LSTM_B", E + H), rec[i], adj[i], n["token"], rec[p] if p is not None else NONE,
                    adj[p] if p is not None else NONE]
        if k == "CS":
            if fwd:
                return [pre("CS_F", len(ch)), rec[i], tok(n["token"])] + [rec[c] for c in ch]
            w = [pre("CS_B", len(ch)), rec[i], adj[i], tok(n["token"])]
            for c in ch:
                w += [rec[c], adj[c]]
            return w
        c = ch[0]
        return ([pre("HEAD_F", H), rec[i], rec[c], n["label"]] if fwd else
                [pre("HEAD_B", H), rec[i], rec[c], adj[c], n["label"]])

    # S4/S5: phases and min-load group assignment
    P = 2 * L + 2
    by_level = [[] for _ in range(L + 1)]
    for i in range(len(nodes)):                  # S4 (R-13): cells first, then heads, ascending global id
        if nodes[i]["kind"] != "HEAD":
            by_level[level[i]].append(i)
    for i in range(len(nodes)):
        if nodes[i]["kind"] == "HEAD":
            by_level[level[i]].append(i)
    graph_group = None
    if by_graph:
        # S5g: whole graphs, longest first (depth, then cell count, then batch index), each to the group
        # whose estimated time after adding it is smallest (ties lowest); time of a group =
        # Σ_levels (2 ceil(n_l / 16) + n_l), n_l = its cells at level l (batches of 16 per level)
        hist = [[0] * (L + 1) for _ in range(len(graphs))]
        for i, n in enumerate(nodes):
            if n["kind"] != "HEAD":
                hist[n["graph"]][level[i]] += 1
        depth = [max((lv for lv in range(L + 1) if hist[b][lv]), default=0) for b in range(len(graphs))]
        order = sorted(range(len(graphs)), key=lambda b: (-depth[b], -sum(hist[b]), b))
        gh = [[0] * (L + 1) for _ in range(G)]

        def est(h):
            return sum(2 * ((x + 15) // 16) + x for x in h)

        graph_group = [0] * len(graphs)
        for b in order:
            g = min(range(G), key=lambda x: (est([a + c for a, c in zip(gh[x], hist[b])]), x))
            gh[g] = [a + c for a, c in zip(gh[g], hist[b])]
            graph_group[b] = g
    phase_instrs = []            # per phase: per group list of words
    part = []
    for p in range(P):
        fwd = p <= L
        lv = p if fwd else 2 * L + 1 - p
        load = [0] * G
        per_g = [[] for _ in range(G)]
        for i in by_level[lv]:
            if by_graph:
                g = graph_group[nodes[i]["graph"]]
            else:
                g = min(range(G), key=lambda x: (load[x], x))
                load[g] += cost(nodes[i])
            per_g[g].extend(instr(i, fwd))
        phase_instrs.append(per_g)
        part.append([g for g in range(G) if per_g[g]])
    # S6: signal / wait
    streams = [[] for _ in range(G)]
    for p in range(P):
        for g in range(G):
            if g not in part[p]:
                continue
            if p >= 1:
                streams[g].append(pre("W", p))
            streams[g].extend(phase_instrs[p][g])
            if p < P - 1:
                streams[g].append(pre("S", p + 1))
    targets = [0] + [n_act * len(part[p - 1]) for p in range(1, n_bar + 1)]
    # §E: header (prefix sums, L169), streams, barrier targets
    prefix = [0]
    for s in streams:
        prefix.append(prefix[-1] + len(s))
    words = [G, n_bar] + prefix
    for s in streams:
        words += s
    words += targets
    return dict(words=[w & 0xFFFFFFFF for w in words], pool_words=pool_words, zero_words=zero_words,
                loss_word=z_loss, n_bar=n_bar, levels=level, nodes=nodes, rec=rec, adj=adj, L=L,
                graph_group=graph_group, G=G, H=H)


DF_OP = dict(LEAF_B=0x21, INT_F=0x22, INT_B=0x23, HEAD_FB=0x42)


def device_lowering(ref):
    """SPEC_SCRIPT.md §D, step by step: the binary cell's device lowering for whole-graph groups (S5g) —
    the gradient GEMM's node lists (L185: one GEMM per matrix over the concatenated operands) and the
    dataflow program of the replica-group kernel (the per-group instruction streams of L141-167 with
    per-node slots in place of the signal/wait of L165).  `ref` is build(..., by_graph=True) of a binary
    batch.  Returns dict(lists: the blob after the SPEC words, df_off: offset of the program inside it,
    n_hx, n_part, n_hd, df_hx, df_part, df_hd, df_words)."""
    nodes, level, rec, adj = ref["nodes"], ref["levels"], ref["rec"], ref["adj"]
    G, L, H, gg = ref["G"], ref["L"], ref["H"], ref["graph_group"]
    NONE_ = NONE
    group = [gg[n["graph"]] for n in nodes]
    # INT list (rec, rec_l, rec_r) and LEAF list (rec, token), grouped by group, ascending global id
    out = []
    for g in range(G):
        for i, n in enumerate(nodes):
            if n["kind"] == "INT" and group[i] == g:
                out += [rec[i], rec[n["children"][0]], rec[n["children"][1]]]
    for g in range(G):
        for i, n in enumerate(nodes):
            if n["kind"] == "LEAF" and group[i] == g:
                out += [rec[i], n["token"]]
    # slots in ascending global id: hx (internal cell with a parent or a head), pp (internal cell),
    # hd (cell with a head); dsrc = pp(parent) << 1 | side
    parent, side, head_of = {}, {}, {}
    for i, n in enumerate(nodes):
        if n["kind"] == "INT":
            for sd, c in enumerate(n["children"]):
                parent[c], side[c] = i, sd
        elif n["kind"] == "HEAD":
            head_of[n["children"][0]] = i
    hx, pp, hd = {}, {}, {}
    for i, n in enumerate(nodes):
        if n["kind"] == "INT" and (i in parent or i in head_of):
            hx[i] = len(hx)
        if n["kind"] == "INT":
            pp[i] = len(pp)
        if i in head_of:
            hd[i] = len(hd)

    def dsrc(i):
        return (pp[parent[i]] << 1 | side[i]) if i in parent else NONE_

    def entry(op, i):
        n = nodes[i]
        if op == "INT_F":
            l, r = n["children"]
            return [rec[i], hx.get(i, NONE_), rec[l], hx.get(l, NONE_), rec[r], hx.get(r, NONE_)]
        if op == "HEAD_FB":
            c = n["children"][0]
            return [rec[i], rec[c], n["label"], hx.get(c, NONE_), hd.get(c, NONE_)]
        if op == "INT_B":
            l, r = n["children"]
            return [rec[i], adj[i], dsrc(i), hd.get(i, NONE_), pp[i], rec[l], adj[l], rec[r], adj[r]]
        return [rec[i], adj[i], dsrc(i), hd.get(i, NONE_)]          # LEAF_B

    def batches(op, ids):
        cap = 64 if op == "LEAF_B" else 16
        w = []
        for b0 in range(0, len(ids), cap):
            chunk = ids[b0:b0 + cap]
            w.append(DF_OP[op] | (len(chunk) << 8))
            for i in chunk:
                w += entry(op, i)
        return w

    progs = []
    for g in range(G):
        w = []
        mine = [i for i in range(len(nodes)) if group[i] == g]
        for lv in range(1, L + 1):                 # forward levels: cells, then the heads of that level
            w += batches("INT_F", [i for i in mine if level[i] == lv and nodes[i]["kind"] == "INT"])
            w += batches("HEAD_FB", [i for i in mine if level[i] == lv and nodes[i]["kind"] == "HEAD"])
        for lv in range(L, -1, -1):                # backward levels in reverse (L167)
            w += batches("INT_B", [i for i in mine if level[i] == lv and nodes[i]["kind"] == "INT"])
            w += batches("LEAF_B", [i for i in mine if level[i] == lv and nodes[i]["kind"] == "LEAF"])
        progs.append(w)
    df_off = len(out)
    pre = [0]
    for w in progs:
        pre.append(pre[-1] + len(w))
    out += [G] + pre
    for w in progs:
        out += w
    # tagged regions behind the SPEC pool: 64-bit slots (2 words), each region aligned to 32 words
    df_hx = _a32(ref["pool_words"])
    df_part = _a32(df_hx + 2 * H * len(hx))
    df_hd = _a32(df_part + 2 * 32 * H * len(pp))
    end = _a32(df_hd + 2 * H * len(hd))
    return dict(lists=[x & 0xFFFFFFFF for x in out], df_off=df_off, n_hx=len(hx), n_part=len(pp), n_hd=len(hd),
                df_hx=df_hx, df_part=df_part, df_hd=df_hd, df_words=end - ref["pool_words"])


def chain_table(graphs, Gd: int, dirs: int):
    """SPEC_SCRIPT.md §L chain recurrence table, step by step: sentences longest first, each to the group with
    the smallest total length among those with fewer than 64 sentences (ties lowest), the table words (direction
    1's groups repeat direction 0's).  None when a sentence finds no group."""
    lens = [len(g) for g in graphs]
    offs = [0]
    for n in lens:
        offs.append(offs[-1] + n)
    order = sorted(range(len(graphs)), key=lambda g: -lens[g])          # stable: ties keep batch order
    mem, load = [[] for _ in range(Gd)], [0] * Gd
    for g in order:
        if lens[g] == 0:
            continue
        cand = [q for q in range(Gd) if len(mem[q]) < 64]
        if not cand:
            return None
        q = min(cand, key=lambda x: (load[x], x))
        mem[q].append(g)
        load[q] += lens[g]
    G = Gd * dirs
    words, pre, run = [G, 0], [], 0
    for q in range(G):
        run += len(mem[q % Gd])
        pre.append(run)
    words += pre
    for q in range(G):
        for g in mem[q % Gd]:
            words += [offs[g], lens[g]]
    return words
