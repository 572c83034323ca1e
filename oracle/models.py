"""Oracle models (TEST INFRASTRUCTURE ONLY — see oracle/__init__.py).

What VPPS computes (in-register caching and scripted scheduling are an
execution strategy and do not change the math).  For parameters θ and a batch of graphs
G_1..G_B the method returns
    L(θ) = Σ_b ℓ_b(θ)                         (super-graph with summed loss, L205)
    ∇_θ L for every matrix and bias, ∇_X L for the caller's input table,
    and in fused mode θ' = θ − η(∇_θ L + λθ)  (parameter update in the same kernel, L129, L197).

The paper gives no cell equations; they follow its refs [4] (LSTM, L320), [5] (Tree-LSTM,
L321) and the readings of SURVEY.md §8(c) c.2 / DESIGN.md "Readings" (R-1 … R-6):
  M1  LSTM step, gates stacked (i, f, o, g):  a = W x + U h_prev + b
  M2  BiLSTM tagger: forward/backward LSTM, m = tanh(W_mlp[h→; h←] + b_mlp), z = W_tag m + b_tag
  M3  child-sum Tree-LSTM ([5] eqs. 2-8), stacked (i, o, u)
  M4  binary Tree-LSTM ([5] eqs. 9-14, N = 2, words at leaves only, diagonal forget couplings),
      matrices W_iou 3H×E, U_iou 3H×2H, U_fl H×H, U_fr H×H, W_out C×H  (11H²+5H at E=H: Tab.I)
  M5  GRU step (Cho et al.; the variation L21 names; reading R-34): gates
      stacked (r, z, n), a_x = W x + b_i, a_h = U h_prev + b_h,
      r = σ(a_x[r] + a_h[r]), z = σ(a_x[z] + a_h[z]), n = tanh(a_x[n] + r ⊙ a_h[n]),
      h = (1 − z) ⊙ n + z ⊙ h_prev
  M6  RvNN (Socher-style recursive net with untied leaf / internal weights; reading R-35):
      leaf h = tanh(W_leaf x + b_leaf), internal h = tanh(W_int [h_l; h_r] + b_int)
  M7  TD-RNN (reading R-36): a DAG over a sentence — level 0 the embeddings themselves
      (h = x, E = H), node i of level k: h = tanh(W [h_i; h_{i+1}] + b) over level k−1 (one composition
      function; inner nodes have two parents), the softmax head on the labelled top node
  M8  TD-LSTM (reading R-37): M4's binary Tree-LSTM cell on the TD-RNN pyramid DAG (leaves are
      M4 leaf cells on the tokens; shared children accumulate dh and dc from both parents)
  M9  BiLSTMwChar (reading R-38): M2 where the embedding of a rare word is [h→_c(last char);
      h←_c(first char)] of a character BiLSTM (hidden E/2 per direction, char embeddings C_emb of
      length Ec = 64, L281) over the word's spelling; a node is (children, tok, label, chars) and a
      non-empty `chars` marks the word rare (its row of X is not read)
  head: z = W_out h + b_out, ℓ = −log softmax(z)[y]  ("negative softmax log likelihood", L42)

Everything is float64, node by node, in the graph's own order for the forward pass and in
reverse order for the hand-written reverse pass (the textbook derivatives of SURVEY.md c.2b).
No batching, fusion or reordering beyond that.
"""
from __future__ import annotations

import numpy as np

CELLS = ("lstm", "binary", "childsum", "bilstm", "gru", "rvnn", "tdrnn", "tdlstm", "bilstmchar")


def param_shapes(cell: str, H: int, E: int, C: int, M: int = 256, Ec: int = 64, Vc: int = 64):
    """Ordered (name, shape) list of a model's parameters: matrices first, then biases.

    This is the parameter order of the C ABI (include/vpps.h, vpps_define_model)."""
    if cell == "lstm":
        return [("W", (4 * H, E)), ("U", (4 * H, H)), ("W_out", (C, H)),
                ("b", (4 * H,)), ("b_out", (C,))]
    if cell in ("binary", "tdlstm"):
        return [("W_iou", (3 * H, E)), ("U_iou", (3 * H, 2 * H)), ("U_fl", (H, H)), ("U_fr", (H, H)),
                ("W_out", (C, H)), ("b_iou", (3 * H,)), ("b_f", (H,)), ("b_out", (C,))]
    if cell == "childsum":
        return [("W_iou", (3 * H, E)), ("W_f", (H, E)), ("U_iou", (3 * H, H)), ("U_f", (H, H)),
                ("W_out", (C, H)), ("b_iou", (3 * H,)), ("b_f", (H,)), ("b_out", (C,))]
    if cell == "tdrnn":
        return [("W", (H, 2 * H)), ("W_out", (C, H)), ("b", (H,)), ("b_out", (C,))]
    if cell == "rvnn":
        return [("W_leaf", (H, E)), ("W_int", (H, 2 * H)), ("W_out", (C, H)),
                ("b_leaf", (H,)), ("b_int", (H,)), ("b_out", (C,))]
    if cell == "gru":
        return [("W", (3 * H, E)), ("U", (3 * H, H)), ("W_out", (C, H)),
                ("b_i", (3 * H,)), ("b_h", (3 * H,)), ("b_out", (C,))]
    if cell == "bilstm":
        return [("Wf", (4 * H, E)), ("Uf", (4 * H, H)), ("Wb", (4 * H, E)), ("Ub", (4 * H, H)),
                ("W_mlp", (M, 2 * H)), ("W_tag", (C, M)),
                ("bf", (4 * H,)), ("bb", (4 * H,)), ("b_mlp", (M,)), ("b_tag", (C,))]
    if cell == "bilstmchar":      # M2 + the character BiLSTM (hidden Hc = E/2 per direction, R-38)
        if E % 2:
            raise ValueError("BiLSTMwChar: E must be even ([h→_c; h←_c] is the rare word's embedding)")
        Hc = E // 2
        return [("Wf", (4 * H, E)), ("Uf", (4 * H, H)), ("Wb", (4 * H, E)), ("Ub", (4 * H, H)),
                ("W_mlp", (M, 2 * H)), ("W_tag", (C, M)),
                ("C_emb", (Vc, Ec)), ("Wcf", (4 * Hc, Ec)), ("Ucf", (4 * Hc, Hc)), ("Wcb", (4 * Hc, Ec)),
                ("Ucb", (4 * Hc, Hc)),
                ("bf", (4 * H,)), ("bb", (4 * H,)), ("b_mlp", (M,)), ("b_tag", (C,)),
                ("bcf", (4 * Hc,)), ("bcb", (4 * Hc,))]
    raise ValueError(cell)


def sigmoid(x):
    return 1.0 / (1.0 + np.exp(-x))


def log_softmax(z):
    m = np.max(z)
    return z - m - np.log(np.sum(np.exp(z - m)))


# ----------------------------------------------------------------------------------------
# loss head (L42): z = W_out h + b_out, ℓ = −log softmax(z)[y];  dz = softmax(z) − onehot(y)
# ----------------------------------------------------------------------------------------
def head_forward(P, h, y, wname="W_out", bname="b_out"):
    z = P[wname] @ h + P[bname]
    ls = log_softmax(z)
    return -ls[y], np.exp(ls)


def head_backward(P, G, h, p, y, wname="W_out", bname="b_out"):
    dz = p.copy()
    dz[y] -= 1.0
    G[wname] += np.outer(dz, h)
    G[bname] += dz
    return P[wname].T @ dz


# ----------------------------------------------------------------------------------------
# M1: LSTM step (Gers et al. [4]; gate order i, f, o, g)
# ----------------------------------------------------------------------------------------
def lstm_step(W, U, b, x, h_prev, c_prev):
    H = U.shape[1]
    a = W @ x + U @ h_prev + b
    i = sigmoid(a[0:H]); f = sigmoid(a[H:2 * H]); o = sigmoid(a[2 * H:3 * H]); g = np.tanh(a[3 * H:4 * H])
    c = f * c_prev + i * g
    h = o * np.tanh(c)
    return dict(i=i, f=f, o=o, g=g, c=c, h=h, x=x, h_prev=h_prev, c_prev=c_prev)


def lstm_step_backward(W, U, s, dh, dc):
    """Returns (γ, dx, dh_prev, dc_prev); γ is the pre-activation gradient [i f o g]."""
    tc = np.tanh(s["c"])
    do = dh * tc
    chat = dc + dh * s["o"] * (1.0 - tc * tc)
    di = chat * s["g"]
    dg = chat * s["i"]
    df = chat * s["c_prev"]
    dc_prev = chat * s["f"]
    gam = np.concatenate([di * s["i"] * (1 - s["i"]), df * s["f"] * (1 - s["f"]),
                          do * s["o"] * (1 - s["o"]), dg * (1 - s["g"] ** 2)])
    return gam, W.T @ gam, U.T @ gam, dc_prev


def _lstm_graph(P, G, X, dX, nodes, H):
    """One LSTM chain (node t's single child is t-1). Returns the graph's loss."""
    n = len(nodes)
    st = [None] * n
    loss = 0.0
    heads = {}
    for t, (ch, tok, lab) in enumerate(nodes):
        hp = st[ch[0]]["h"] if ch else np.zeros(H)
        cp = st[ch[0]]["c"] if ch else np.zeros(H)
        st[t] = lstm_step(P["W"], P["U"], P["b"], X[tok], hp, cp)
        if lab >= 0:
            l, p = head_forward(P, st[t]["h"], lab)
            loss += l
            heads[t] = p
    dh = [np.zeros(H) for _ in range(n)]
    dc = [np.zeros(H) for _ in range(n)]
    for t in range(n - 1, -1, -1):
        ch, tok, lab = nodes[t]
        if lab >= 0:
            dh[t] += head_backward(P, G, st[t]["h"], heads[t], lab)
        gam, dx, dhp, dcp = lstm_step_backward(P["W"], P["U"], st[t], dh[t], dc[t])
        G["W"] += np.outer(gam, st[t]["x"])
        G["U"] += np.outer(gam, st[t]["h_prev"])
        G["b"] += gam
        dX[tok] += dx
        if ch:
            dh[ch[0]] += dhp
            dc[ch[0]] += dcp
    return loss


# ----------------------------------------------------------------------------------------
# M5: GRU step (gate order r, z, n; the reset gate multiplies U_n h_prev + b_hn, reading R-34)
# ----------------------------------------------------------------------------------------
def gru_step(W, U, b_i, b_h, x, h_prev):
    H = U.shape[1]
    ax = W @ x + b_i
    ah = U @ h_prev + b_h
    r = sigmoid(ax[0:H] + ah[0:H])
    z = sigmoid(ax[H:2 * H] + ah[H:2 * H])
    n = np.tanh(ax[2 * H:3 * H] + r * ah[2 * H:3 * H])
    h = (1.0 - z) * n + z * h_prev
    return dict(r=r, z=z, n=n, hn=ah[2 * H:3 * H], h=h, x=x, h_prev=h_prev)


def gru_step_backward(W, U, s, dh):
    """Returns (γ_x, γ_h, dx, dh_prev): γ_x the gradient of a_x = W x + b_i, γ_h that of a_h = U h + b_h."""
    r, z, n = s["r"], s["z"], s["n"]
    dn = dh * (1.0 - z)
    dz = dh * (s["h_prev"] - n)
    dan = dn * (1.0 - n * n)                 # pre-activation of n
    dr = dan * s["hn"]
    dar = dr * r * (1.0 - r)
    daz = dz * z * (1.0 - z)
    gam_x = np.concatenate([dar, daz, dan])
    gam_h = np.concatenate([dar, daz, dan * r])
    return gam_x, gam_h, W.T @ gam_x, U.T @ gam_h + dh * z


def _gru_graph(P, G, X, dX, nodes, H):
    """One GRU chain (node t's single child is t-1). Returns the graph's loss."""
    n = len(nodes)
    st = [None] * n
    loss = 0.0
    heads = {}
    for t, (ch, tok, lab) in enumerate(nodes):
        hp = st[ch[0]]["h"] if ch else np.zeros(H)
        st[t] = gru_step(P["W"], P["U"], P["b_i"], P["b_h"], X[tok], hp)
        if lab >= 0:
            l, p = head_forward(P, st[t]["h"], lab)
            loss += l
            heads[t] = p
    dh = [np.zeros(H) for _ in range(n)]
    for t in range(n - 1, -1, -1):
        ch, tok, lab = nodes[t]
        if lab >= 0:
            dh[t] += head_backward(P, G, st[t]["h"], heads[t], lab)
        gx, gh, dx, dhp = gru_step_backward(P["W"], P["U"], st[t], dh[t])
        G["W"] += np.outer(gx, st[t]["x"])
        G["U"] += np.outer(gh, st[t]["h_prev"])
        G["b_i"] += gx
        G["b_h"] += gh
        dX[tok] += dx
        if ch:
            dh[ch[0]] += dhp
    return loss


# ----------------------------------------------------------------------------------------
# M6: RvNN (untied leaf / internal transformations, reading R-35)
# ----------------------------------------------------------------------------------------
def _rvnn_graph(P, G, X, dX, nodes, H):
    """One binary tree: leaves carry a token, internal nodes two children. Returns the graph's loss."""
    n = len(nodes)
    h = [None] * n
    loss = 0.0
    heads = {}
    for v, (ch, tok, lab) in enumerate(nodes):
        if not ch:
            h[v] = np.tanh(P["W_leaf"] @ X[tok] + P["b_leaf"])
        else:
            h[v] = np.tanh(P["W_int"] @ np.concatenate([h[ch[0]], h[ch[1]]]) + P["b_int"])
        if lab >= 0:
            l, p = head_forward(P, h[v], lab)
            loss += l
            heads[v] = p
    dh = [np.zeros(H) for _ in range(n)]
    for v in range(n - 1, -1, -1):
        ch, tok, lab = nodes[v]
        if lab >= 0:
            dh[v] += head_backward(P, G, h[v], heads[v], lab)
        g = dh[v] * (1.0 - h[v] * h[v])              # pre-activation gradient
        if not ch:
            G["W_leaf"] += np.outer(g, X[tok])
            G["b_leaf"] += g
            dX[tok] += P["W_leaf"].T @ g
        else:
            x = np.concatenate([h[ch[0]], h[ch[1]]])
            G["W_int"] += np.outer(g, x)
            G["b_int"] += g
            dx = P["W_int"].T @ g
            dh[ch[0]] += dx[:H]
            dh[ch[1]] += dx[H:]
    return loss


# ----------------------------------------------------------------------------------------
# M7: TD-RNN (reading R-36): leaves are the embeddings, one composition function, shared children
# ----------------------------------------------------------------------------------------
def _tdrnn_graph(P, G, X, dX, nodes, H):
    n = len(nodes)
    h = [None] * n
    loss = 0.0
    heads = {}
    for v, (ch, tok, lab) in enumerate(nodes):
        h[v] = X[tok].copy() if not ch else np.tanh(P["W"] @ np.concatenate([h[ch[0]], h[ch[1]]]) + P["b"])
        if lab >= 0:
            l, p = head_forward(P, h[v], lab)
            loss += l
            heads[v] = p
    dh = [np.zeros(H) for _ in range(n)]
    for v in range(n - 1, -1, -1):         # every parent of v comes after v: its dh is complete here
        ch, tok, lab = nodes[v]
        if lab >= 0:
            dh[v] += head_backward(P, G, h[v], heads[v], lab)
        if not ch:
            dX[tok] += dh[v]
            continue
        g = dh[v] * (1.0 - h[v] * h[v])
        G["W"] += np.outer(g, np.concatenate([h[ch[0]], h[ch[1]]]))
        G["b"] += g
        dx = P["W"].T @ g
        dh[ch[0]] += dx[:H]
        dh[ch[1]] += dx[H:]
    return loss


# ----------------------------------------------------------------------------------------
# M4: binary Tree-LSTM ([5] eqs. 9-14 with N = 2; stacked rows [i; o; u])
# ----------------------------------------------------------------------------------------
def _binary_graph(P, G, X, dX, nodes, H):
    n = len(nodes)
    st = [None] * n
    loss = 0.0
    heads = {}
    for v, (ch, tok, lab) in enumerate(nodes):
        if len(ch) == 0:
            x = X[tok]
            a = P["W_iou"] @ x + P["b_iou"]
            i = sigmoid(a[:H]); o = sigmoid(a[H:2 * H]); u = np.tanh(a[2 * H:])
            c = i * u
            st[v] = dict(i=i, o=o, u=u, c=c, h=o * np.tanh(c), x=x)
        else:
            l, r = ch
            hl, hr = st[l]["h"], st[r]["h"]
            a = P["U_iou"] @ np.concatenate([hl, hr]) + P["b_iou"]
            i = sigmoid(a[:H]); o = sigmoid(a[H:2 * H]); u = np.tanh(a[2 * H:])
            fl = sigmoid(P["U_fl"] @ hl + P["b_f"])
            fr = sigmoid(P["U_fr"] @ hr + P["b_f"])
            c = i * u + fl * st[l]["c"] + fr * st[r]["c"]
            st[v] = dict(i=i, o=o, u=u, fl=fl, fr=fr, c=c, h=o * np.tanh(c))
        if lab >= 0:
            lv, p = head_forward(P, st[v]["h"], lab)
            loss += lv
            heads[v] = p
    dh = [np.zeros(H) for _ in range(n)]
    dc = [np.zeros(H) for _ in range(n)]
    for v in range(n - 1, -1, -1):
        ch, tok, lab = nodes[v]
        s = st[v]
        if lab >= 0:
            dh[v] += head_backward(P, G, s["h"], heads[v], lab)
        t = np.tanh(s["c"])
        do = dh[v] * t
        chat = dc[v] + dh[v] * s["o"] * (1.0 - t * t)
        di = chat * s["u"]
        du = chat * s["i"]
        g = np.concatenate([di * s["i"] * (1 - s["i"]), do * s["o"] * (1 - s["o"]), du * (1 - s["u"] ** 2)])
        G["b_iou"] += g
        if len(ch) == 0:
            G["W_iou"] += np.outer(g, s["x"])
            dX[tok] += P["W_iou"].T @ g
        else:
            l, r = ch
            hl, hr = st[l]["h"], st[r]["h"]
            gfl = chat * st[l]["c"] * s["fl"] * (1 - s["fl"])
            gfr = chat * st[r]["c"] * s["fr"] * (1 - s["fr"])
            dc[l] += chat * s["fl"]
            dc[r] += chat * s["fr"]
            G["b_f"] += gfl + gfr
            G["U_iou"] += np.outer(g, np.concatenate([hl, hr]))
            G["U_fl"] += np.outer(gfl, hl)
            G["U_fr"] += np.outer(gfr, hr)
            dlr = P["U_iou"].T @ g
            dh[l] += dlr[:H] + P["U_fl"].T @ gfl
            dh[r] += dlr[H:] + P["U_fr"].T @ gfr
    return loss


# ----------------------------------------------------------------------------------------
# M3: child-sum Tree-LSTM ([5] eqs. 2-8; stacked rows [i; o; u]; optional word at any node)
# ----------------------------------------------------------------------------------------
def _childsum_graph(P, G, X, dX, nodes, H):
    n = len(nodes)
    E = P["W_iou"].shape[1]
    st = [None] * n
    loss = 0.0
    heads = {}
    for v, (ch, tok, lab) in enumerate(nodes):
        x = X[tok] if tok >= 0 else np.zeros(E)
        hsum = np.zeros(H)
        for k in ch:
            hsum = hsum + st[k]["h"]
        a = P["W_iou"] @ x + P["U_iou"] @ hsum + P["b_iou"]
        i = sigmoid(a[:H]); o = sigmoid(a[H:2 * H]); u = np.tanh(a[2 * H:])
        fx = P["W_f"] @ x + P["b_f"]
        fs = [sigmoid(fx + P["U_f"] @ st[k]["h"]) for k in ch]
        c = i * u
        for f, k in zip(fs, ch):
            c = c + f * st[k]["c"]
        st[v] = dict(i=i, o=o, u=u, f=fs, c=c, h=o * np.tanh(c), x=x, hsum=hsum)
        if lab >= 0:
            lv, p = head_forward(P, st[v]["h"], lab)
            loss += lv
            heads[v] = p
    dh = [np.zeros(H) for _ in range(n)]
    dc = [np.zeros(H) for _ in range(n)]
    for v in range(n - 1, -1, -1):
        ch, tok, lab = nodes[v]
        s = st[v]
        if lab >= 0:
            dh[v] += head_backward(P, G, s["h"], heads[v], lab)
        t = np.tanh(s["c"])
        do = dh[v] * t
        chat = dc[v] + dh[v] * s["o"] * (1.0 - t * t)
        g = np.concatenate([chat * s["u"] * s["i"] * (1 - s["i"]), do * s["o"] * (1 - s["o"]),
                            chat * s["i"] * (1 - s["u"] ** 2)])
        G["b_iou"] += g
        G["W_iou"] += np.outer(g, s["x"])
        G["U_iou"] += np.outer(g, s["hsum"])
        dx = P["W_iou"].T @ g
        dhs = P["U_iou"].T @ g
        for f, k in zip(s["f"], ch):
            gf = chat * st[k]["c"] * f * (1 - f)
            dc[k] += chat * f
            dh[k] += dhs + P["U_f"].T @ gf
            G["U_f"] += np.outer(gf, st[k]["h"])
            G["W_f"] += np.outer(gf, s["x"])
            G["b_f"] += gf
            dx = dx + P["W_f"].T @ gf
        if tok >= 0:
            dX[tok] += dx
    return loss


# ----------------------------------------------------------------------------------------
# M2: BiLSTM tagger ([25] via L265, L281): positions t = 0..n-1 of a chain
# ----------------------------------------------------------------------------------------
def _bilstm_graph(P, G, X, dX, nodes, H):
    toks = [nd[1] for nd in nodes]
    loss, dxs = _bilstm_core(P, G, [X[k] for k in toks], nodes, H)
    for t, k in enumerate(toks):
        dX[k] += dxs[t]
    return loss


def _bilstm_core(P, G, xs, nodes, H):
    """M2 over the word vectors xs[t]: summed loss, parameter gradients into G, returns dL/dxs[t]."""
    n = len(nodes)
    sf, sb = [None] * n, [None] * n
    h, c = np.zeros(H), np.zeros(H)
    for t in range(n):
        sf[t] = lstm_step(P["Wf"], P["Uf"], P["bf"], xs[t], h, c)
        h, c = sf[t]["h"], sf[t]["c"]
    h, c = np.zeros(H), np.zeros(H)
    for t in range(n - 1, -1, -1):
        sb[t] = lstm_step(P["Wb"], P["Ub"], P["bb"], xs[t], h, c)
        h, c = sb[t]["h"], sb[t]["c"]
    loss = 0.0
    dhf = [np.zeros(H) for _ in range(n)]
    dhb = [np.zeros(H) for _ in range(n)]
    for t, nd in enumerate(nodes):
        lab = nd[2]
        if lab < 0:
            continue
        hcat = np.concatenate([sf[t]["h"], sb[t]["h"]])
        m = np.tanh(P["W_mlp"] @ hcat + P["b_mlp"])
        lv, p = head_forward(P, m, lab, "W_tag", "b_tag")
        loss += lv
        dm = head_backward(P, G, m, p, lab, "W_tag", "b_tag")
        da = dm * (1 - m * m)
        G["W_mlp"] += np.outer(da, hcat)
        G["b_mlp"] += da
        dcat = P["W_mlp"].T @ da
        dhf[t] += dcat[:H]
        dhb[t] += dcat[H:]
    dxs = [None] * n
    dh, dc = np.zeros(H), np.zeros(H)
    for t in range(n - 1, -1, -1):
        gam, dx, dh, dc = lstm_step_backward(P["Wf"], P["Uf"], sf[t], dhf[t] + dh, dc)
        G["Wf"] += np.outer(gam, sf[t]["x"]); G["Uf"] += np.outer(gam, sf[t]["h_prev"]); G["bf"] += gam
        dxs[t] = dx
    dh, dc = np.zeros(H), np.zeros(H)
    for t in range(n):
        gam, dx, dh, dc = lstm_step_backward(P["Wb"], P["Ub"], sb[t], dhb[t] + dh, dc)
        G["Wb"] += np.outer(gam, sb[t]["x"]); G["Ub"] += np.outer(gam, sb[t]["h_prev"]); G["bb"] += gam
        dxs[t] = dxs[t] + dx
    return loss, dxs


def _char_encode(P, chars):
    """M9 character BiLSTM over one word's spelling: returns [h→(last); h←(first)] and the
    recorded steps of both directions."""
    Hc = P["Ucf"].shape[1]
    n = len(chars)
    sf, sb = [None] * n, [None] * n
    h, c = np.zeros(Hc), np.zeros(Hc)
    for t in range(n):
        sf[t] = lstm_step(P["Wcf"], P["Ucf"], P["bcf"], P["C_emb"][chars[t]], h, c)
        h, c = sf[t]["h"], sf[t]["c"]
    h, c = np.zeros(Hc), np.zeros(Hc)
    for t in range(n - 1, -1, -1):
        sb[t] = lstm_step(P["Wcb"], P["Ucb"], P["bcb"], P["C_emb"][chars[t]], h, c)
        h, c = sb[t]["h"], sb[t]["c"]
    return np.concatenate([sf[n - 1]["h"], sb[0]["h"]]), (sf, sb)


def _char_backward(P, G, chars, rec, drep):
    """Reverse of _char_encode: dL/drep enters at the forward direction's last step and the backward
    direction's last-processed (first-char) step only."""
    Hc = P["Ucf"].shape[1]
    sf, sb = rec
    n = len(chars)
    dh, dc = drep[:Hc].copy(), np.zeros(Hc)
    for t in range(n - 1, -1, -1):
        gam, dx, dh, dc = lstm_step_backward(P["Wcf"], P["Ucf"], sf[t], dh, dc)
        G["Wcf"] += np.outer(gam, sf[t]["x"]); G["Ucf"] += np.outer(gam, sf[t]["h_prev"]); G["bcf"] += gam
        G["C_emb"][chars[t]] += dx
    dh, dc = drep[Hc:].copy(), np.zeros(Hc)
    for t in range(n):
        gam, dx, dh, dc = lstm_step_backward(P["Wcb"], P["Ucb"], sb[t], dh, dc)
        G["Wcb"] += np.outer(gam, sb[t]["x"]); G["Ucb"] += np.outer(gam, sb[t]["h_prev"]); G["bcb"] += gam
        G["C_emb"][chars[t]] += dx


def _bilstmchar_graph(P, G, X, dX, nodes, H):
    """M9: rare words (non-empty chars) take the character BiLSTM's output as their embedding."""
    xs, recs = [], []
    for nd in nodes:
        chars = nd[3] if len(nd) > 3 else ()
        if chars:
            rep, rec = _char_encode(P, chars)
            xs.append(rep); recs.append(rec)
        else:
            xs.append(X[nd[1]]); recs.append(None)
    loss, dxs = _bilstm_core(P, G, xs, nodes, H)
    for t, nd in enumerate(nodes):
        if recs[t] is None:
            dX[nd[1]] += dxs[t]
        else:
            _char_backward(P, G, nd[3], recs[t], dxs[t])
    return loss


_GRAPH_FN = {"lstm": _lstm_graph, "binary": _binary_graph, "childsum": _childsum_graph,
             "bilstm": _bilstm_graph, "gru": _gru_graph, "rvnn": _rvnn_graph, "tdrnn": _tdrnn_graph,
             "tdlstm": _binary_graph, "bilstmchar": _bilstmchar_graph}   # M4's reverse pass accumulates dh / dc (+=): correct on DAGs


def validate(cell: str, graphs, n_tokens: int, n_classes: int, n_chars: int = 0):
    """Structural rules of the op sets (readings R-4, R-26); raises ValueError."""
    for nodes in graphs:
        for v, nd in enumerate(nodes):
            ch, tok, lab = nd[:3]
            if len(nd) > 3 and (cell != "bilstmchar" or any(not (0 <= k < n_chars) for k in nd[3])):
                raise ValueError("a character spelling needs cell 'bilstmchar' and ids in [0, n_chars)")
            if any(not (0 <= k < v) for k in ch):
                raise ValueError("children must precede their parent")
            if not (-1 <= tok < n_tokens) or not (-1 <= lab < n_classes):
                raise ValueError("token/label out of range")
            if cell in ("binary", "rvnn", "tdrnn", "tdlstm") and not ((len(ch) == 0 and tok >= 0) or (len(ch) == 2 and tok < 0)):
                raise ValueError("binary Tree-LSTM: leaves carry a token, internal nodes have 2 children")
            if cell in ("lstm", "bilstm", "gru", "bilstmchar") and (len(ch) > 1 or tok < 0 or (ch and ch[0] != v - 1)):
                raise ValueError("LSTM chain: node t has child t-1 and a token")
        parents = [0] * len(nodes)
        for nd in nodes:
            for k in nd[0]:
                parents[k] += 1
        if cell not in ("tdrnn", "tdlstm") and any(p > 1 for p in parents):   # TD graphs are DAGs (R-36/37)
            raise ValueError("a node may have at most one parent")


def forward_backward(cell: str, P: dict, X: np.ndarray, graphs, H: int):
    """Summed loss of the batch, gradients of every parameter, gradient of the input table."""
    P = {k: np.asarray(v, dtype=np.float64) for k, v in P.items()}
    X = np.asarray(X, dtype=np.float64)
    G = {k: np.zeros_like(v) for k, v in P.items()}
    dX = np.zeros_like(X)
    loss = 0.0
    for nodes in graphs:       # super-graph = disjoint union, aggregated loss = sum (L205)
        loss += _GRAPH_FN[cell](P, G, X, dX, nodes, H)
    return loss, G, dX


def sgd(P: dict, G: dict, lr: float, weight_decay: float):
    """θ' = θ − η(g + λθ): 'apply gradients' with the model's weight decay (L129, L197; R-6)."""
    return {k: P[k] - lr * (G[k] + weight_decay * P[k]) for k in P}


def flop_count(cell: str, graphs, H: int, E: int, C: int, want_dx: bool = True, M: int = 256, Ec_: int = 64):
    """Algorithmic FLOPs of one training pass: 2 per MAC, ×3 per matrix use
    (forward, dW, dx), ×2 where the input gradient is not needed."""
    f = 0
    kx = 3 if want_dx else 2
    for nodes in graphs:
        if cell == "bilstmchar":
            # M9 (R-38): the word tagger (M2) plus, per rare word of n characters, the character BiLSTM
            # (Hc = E/2 per direction over Ec-wide character embeddings; dx to C_emb needed: x3)
            Hc, Ec = E // 2, Ec_
            f += flop_count("bilstm", [[nd[:3] for nd in nodes]], H, E, C, want_dx, M)
            for nd in nodes:
                n = len(nd[3]) if len(nd) > 3 else 0
                if n:
                    f += 2 * (2 * 4 * Hc * Ec * 3 * n + 2 * 3 * 4 * Hc * Hc * (n - 1))
            continue
        if cell == "bilstm":
            # M2 (L265, L281): per position and direction the input product (W x) and, after the first
            # step of that direction, the recurrent product (U h); per labelled position the MLP over
            # [h_fwd; h_bwd] (M x 2H) and the tag head (C x M); no MLP or head where there is no label
            n = len(nodes)
            f += 2 * (2 * 4 * H * E * kx * n + 2 * 3 * 4 * H * H * max(n - 1, 0))
            f += sum(2 * 3 * (M * 2 * H + C * M) for nd in nodes if nd[2] >= 0)
            continue
        for nd in nodes:
            ch, tok, lab = nd[:3]
            if cell in ("binary", "tdlstm"):
                f += (2 * 3 * H * E * kx) if not ch else 2 * 3 * (3 * H * 2 * H + 2 * H * H)
            elif cell == "childsum":
                k = len(ch)
                mac_x = 4 * H * E if tok >= 0 else 0      # W_iou x and W_f x (once per node)
                f += 2 * mac_x * kx
                f += 2 * 3 * (3 * H * H + k * H * H) if k else 0
            elif cell == "lstm":
                f += 2 * (4 * H * E) * kx + 2 * 3 * 4 * H * H * (1 if ch else 0)
            elif cell == "tdrnn":
                f += 0 if not ch else 2 * 3 * H * 2 * H
            elif cell == "rvnn":
                f += (2 * H * E * kx) if not ch else 2 * 3 * H * 2 * H
            elif cell == "gru":
                f += 2 * (3 * H * E) * kx + 2 * 3 * 3 * H * H * (1 if ch else 0)
            if lab >= 0 and cell != "bilstm":
                f += 2 * 3 * C * H
    return f
