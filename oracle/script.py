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
                loss_word=z_loss, n_bar=n_bar, levels=level, nodes=nodes, rec=rec, adj=adj)
