"""Pins of the oracle models against things other than themselves (CPU only).

  * brute force: central finite differences in float64 on tiny graphs (every cell, every param)
  * library special cases: torch.nn.LSTMCell / nn.LSTM / cross_entropy in float64
      - M1 chain == torch LSTMCell chain (+ cross-entropy head)
      - M4 on a left-comb (right-comb) tree with zero-embedding side leaves == torch LSTMCell chain
        (pins gate order [i;o;u], which half of U_iou / which of U_fl,U_fr meets which child)
      - M2 == torch nn.LSTM(bidirectional=True) + Linear/tanh/Linear + cross-entropy
  * invariants: M3 on a chain == M1 with stacked [W_i;W_f;W_o;W_u]; batch-order invariance;
    duplicated graph doubles loss and gradients
  * paper values: Tab.I from the M4 parameter inventory
  * closed forms: single-leaf h, softmax-NLL gradient, SGD with weight decay
"""
import math
import os

import numpy as np
import pytest
import torch

import synth
from oracle import models as M

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _params(cell, H, E, C, seed=0, M_=4, **kw):
    rng = np.random.default_rng(seed)
    return synth.init_params(M.param_shapes(cell, H, E, C, M_, **kw), rng)


def _fd_check(cell, graphs, H, E, C, V, M_=4, eps=1e-6, tol=1e-7, **kw):
    rng = np.random.default_rng(1)
    P = _params(cell, H, E, C, 2, M_, **kw)
    # larger weights so that every gate is away from saturation-free linear regime
    P = {k: v * 3.0 for k, v in P.items()}
    X = rng.uniform(-1, 1, size=(V, E))
    loss, G, dX = M.forward_backward(cell, P, X, graphs, H)
    for name in P:
        flat = P[name].reshape(-1)
        for idx in range(flat.size):
            old = flat[idx]
            flat[idx] = old + eps
            lp = M.forward_backward(cell, P, X, graphs, H)[0]
            flat[idx] = old - eps
            lm = M.forward_backward(cell, P, X, graphs, H)[0]
            flat[idx] = old
            num = (lp - lm) / (2 * eps)
            assert abs(num - G[name].reshape(-1)[idx]) < tol * max(1.0, abs(num)), (cell, name, idx)
    for r in range(V):
        for c in range(E):
            old = X[r, c]
            X[r, c] = old + eps
            lp = M.forward_backward(cell, P, X, graphs, H)[0]
            X[r, c] = old - eps
            lm = M.forward_backward(cell, P, X, graphs, H)[0]
            X[r, c] = old
            assert abs((lp - lm) / (2 * eps) - dX[r, c]) < tol * max(1.0, abs(dX[r, c])), (cell, "X", r, c)


def test_fd_binary():
    g1 = [((), 0, -1), ((), 1, -1), ((0, 1), -1, -1), ((), 2, -1), ((2, 3), -1, 1)]
    g2 = [((), 1, -1), ((), 1, -1), ((0, 1), -1, 2)]
    _fd_check("binary", [g1, g2], H=3, E=2, C=3, V=3)


def test_fd_childsum():
    g1 = [((), 0, -1), ((), -1, -1), ((0, 1), 2, -1), ((), 1, -1), ((2, 3), -1, 1)]
    g2 = [((), 1, -1), ((0,), 0, -1), ((1,), -1, 0), ((), 2, -1), ((), 0, -1), ((2, 3, 4), 1, 2)]
    _fd_check("childsum", [g1, g2], H=3, E=2, C=3, V=3)


def test_fd_lstm():
    g1 = [((), 0, 1), ((0,), 2, -1), ((1,), 1, 0)]
    g2 = [((), 1, 2), ((0,), 1, 1)]
    _fd_check("lstm", [g1, g2], H=3, E=2, C=3, V=3)


def test_fd_bilstm():
    g1 = [((), 0, 1), ((0,), 2, -1), ((1,), 1, 0)]
    g2 = [((), 1, 2), ((0,), 1, 1)]
    _fd_check("bilstm", [g1, g2], H=2, E=2, C=3, V=3, M_=3)


def test_fd_gru():
    g1 = [((), 0, 1), ((0,), 2, -1), ((1,), 1, 0)]
    g2 = [((), 1, 2), ((0,), 1, 1)]
    _fd_check("gru", [g1, g2], H=3, E=2, C=3, V=3)


def test_fd_rvnn():
    g1 = [((), 0, -1), ((), 1, -1), ((0, 1), -1, -1), ((), 2, -1), ((2, 3), -1, 1)]
    g2 = [((), 1, -1), ((), 1, -1), ((0, 1), -1, 2)]
    _fd_check("rvnn", [g1, g2], H=3, E=2, C=3, V=3)


def test_rvnn_left_comb_equals_torch_rnncell():
    """M6 on a left-comb tree == torch.nn.RNNCell over the leaf outputs (reading R-35): internal node k has
    the previous node on the left and leaf k on the right, so h_k = tanh(W_hh h_{k-1} + W_ih z_k + b) with
    W_int = [W_hh | W_ih] and z_k = tanh(W_leaf x_k + b_leaf) (torch Linear + tanh); the first state is the
    leftmost leaf's output.  Swapped halves of W_int, a wrong child order or a dropped tanh' fail this."""
    H, E, C, V, n = 4, 3, 5, 6, 5
    P = {k: v * 2.0 for k, v in _params("rvnn", H, E, C, 7).items()}
    rng = np.random.default_rng(8)
    X = rng.uniform(-1, 1, (V, E))
    toks = [int(t) for t in rng.integers(0, V, n)]
    nodes = [((), toks[0], -1)]
    prev = 0
    for k in range(1, n):
        nodes.append(((), toks[k], -1))
        nodes.append(((prev, len(nodes) - 1), -1, -1))
        prev = len(nodes) - 1
    nodes[-1] = (nodes[-1][0], -1, 3)
    loss, G, dX = M.forward_backward("rvnn", P, X, [nodes], H)
    leaf = torch.nn.Linear(E, H, dtype=torch.float64)
    cell = torch.nn.RNNCell(H, H, nonlinearity="tanh", dtype=torch.float64)
    with torch.no_grad():
        leaf.weight.copy_(torch.tensor(P["W_leaf"])); leaf.bias.copy_(torch.tensor(P["b_leaf"]))
        cell.weight_hh.copy_(torch.tensor(P["W_int"][:, :H])); cell.weight_ih.copy_(torch.tensor(P["W_int"][:, H:]))
        cell.bias_ih.copy_(torch.tensor(P["b_int"])); cell.bias_hh.zero_()
    Wo = torch.tensor(P["W_out"], requires_grad=True)
    bo = torch.tensor(P["b_out"], requires_grad=True)
    Xt = torch.tensor(np.array([X[t] for t in toks]), requires_grad=True)
    z = torch.tanh(leaf(Xt))
    h = z[0:1]
    for k in range(1, n):
        h = cell(z[k:k + 1], h)
    ref = torch.nn.functional.cross_entropy((h[0] @ Wo.T + bo)[None], torch.tensor([3]), reduction="sum")
    ref.backward()
    assert abs(loss - ref.item()) < 1e-12
    np.testing.assert_allclose(G["W_int"], np.concatenate([cell.weight_hh.grad.numpy(), cell.weight_ih.grad.numpy()], 1),
                               atol=1e-12)
    np.testing.assert_allclose(G["b_int"], cell.bias_ih.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["W_leaf"], leaf.weight.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["b_leaf"], leaf.bias.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["W_out"], Wo.grad.numpy(), atol=1e-12)
    dXref = np.zeros_like(X)
    for k, t in enumerate(toks):
        dXref[t] += Xt.grad.numpy()[k]
    np.testing.assert_allclose(dX, dXref, atol=1e-12)


def test_fd_tdrnn():
    rng = np.random.default_rng(3)
    g1 = synth.td_pyramid(rng, 4, 3, 3)
    g2 = synth.td_pyramid(rng, 3, 3, 3)
    _fd_check("tdrnn", [g1, g2], H=2, E=2, C=3, V=3)


def test_tdrnn_pyramid_equals_torch_conv1d():
    """M7 (reading R-36) == repeated torch conv1d with kernel 2 (+ tanh) until one position remains: the
    composition W [h_i; h_{i+1}] + b is a kernel-2 convolution with taps W[:, :H], W[:, H:].  The oracle
    walks the DAG node by node and accumulates each shared child's dh from both parents; a dropped parent,
    swapped taps or a wrong tanh' fail this (loss, dW, db, dW_out and dX to 1e-12 in float64)."""
    H, C, V = 4, 5, 9
    P = {k: v * 1.5 for k, v in _params("tdrnn", H, H, C, 5).items()}
    rng = np.random.default_rng(6)
    X = rng.uniform(-1, 1, (V, H))
    graphs = [synth.td_pyramid(rng, n, V, C) for n in (6, 1, 3)]
    loss, G, dX = M.forward_backward("tdrnn", P, X, graphs, H)
    W = torch.tensor(P["W"], requires_grad=True)
    b = torch.tensor(P["b"], requires_grad=True)
    Wo = torch.tensor(P["W_out"], requires_grad=True)
    bo = torch.tensor(P["b_out"], requires_grad=True)
    Xt = torch.tensor(X, requires_grad=True)
    ker = torch.stack([W[:, :H], W[:, H:]], dim=2)          # [H_out, H_in, 2]
    ref = torch.zeros((), dtype=torch.float64)
    for nodes in graphs:
        toks = [t for (ch, t, _) in nodes if not ch]
        e = Xt[toks].T[None]                                # [1, H, n]
        while e.shape[2] > 1:
            e = torch.tanh(torch.nn.functional.conv1d(e, ker, b))
        y = [lab for (_, _, lab) in nodes if lab >= 0][0]
        ref = ref + torch.nn.functional.cross_entropy((e[0, :, 0] @ Wo.T + bo)[None], torch.tensor([y]), reduction="sum")
    ref.backward()
    assert abs(loss - ref.item()) < 1e-12
    np.testing.assert_allclose(G["W"], W.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["b"], b.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["W_out"], Wo.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["b_out"], bo.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(dX, Xt.grad.numpy(), atol=1e-12)


def _unshare(nodes):
    """Tree expansion of a DAG: every use of a shared node gets its own copy of its sub-DAG."""
    out = []

    def emit(v):
        ch, tok, lab = nodes[v]
        kids = tuple(emit(k) for k in ch)
        out.append((kids, tok, -1))
        return len(out) - 1

    top = [v for v, (_, _, lab) in enumerate(nodes) if lab >= 0][0]
    root = emit(top)
    out[root] = (out[root][0], out[root][1], nodes[top][2])
    return out


def test_tdlstm_dag_equals_its_tree_expansion():
    """M8 (reading R-37): the binary Tree-LSTM on a TD pyramid DAG equals M4 on the DAG's tree expansion
    (each shared node duplicated per use) — loss, every weight gradient and dX are sums over the copies, so a
    shared child that kept only one parent's dh or dc fails this.  M4 itself is pinned against torch LSTMCell
    (test_binary_comb_equals_torch_lstmcell)."""
    H, E, C, V = 3, 2, 4, 6
    P = _params("binary", H, E, C, 13)
    rng = np.random.default_rng(14)
    X = rng.uniform(-1, 1, (V, E))
    dags = [synth.td_pyramid(rng, n, V, C) for n in (4, 2, 5)]
    l1, G1, dX1 = M.forward_backward("tdlstm", P, X, dags, H)
    l2, G2, dX2 = M.forward_backward("binary", P, X, [_unshare(g) for g in dags], H)
    assert abs(l1 - l2) < 1e-12
    for k in G1:
        np.testing.assert_allclose(G1[k], G2[k], atol=1e-12)
    np.testing.assert_allclose(dX1, dX2, atol=1e-12)


def test_fd_bilstmchar():
    """M9: every parameter incl. the character BiLSTM and C_emb, and X (rare positions must not touch X:
    word 1 is spelled at every occurrence in g1, so X[1] gets only g2's plain occurrence)."""
    g1 = [((), 0, 1, ()), ((0,), 1, -1, (2, 0, 1)), ((1,), 2, 0, ()), ((2,), 1, 2, (2, 0, 1))]
    g2 = [((), 1, 2, ()), ((0,), 2, 1, (1,))]
    _fd_check("bilstmchar", [g1, g2], H=2, E=4, C=3, V=3, M_=3, Ec=2, Vc=3)


def _torch_bilstm(Wf, Uf, bf, Wb, Ub, bb, H):
    lstm = torch.nn.LSTM(Wf.shape[1], H, bidirectional=True, dtype=torch.float64)
    with torch.no_grad():
        lstm.weight_ih_l0.copy_(torch.tensor(_ifog_to_torch(Wf, H)))
        lstm.weight_hh_l0.copy_(torch.tensor(_ifog_to_torch(Uf, H)))
        lstm.bias_ih_l0.copy_(torch.tensor(_ifog_to_torch(bf, H))); lstm.bias_hh_l0.zero_()
        lstm.weight_ih_l0_reverse.copy_(torch.tensor(_ifog_to_torch(Wb, H)))
        lstm.weight_hh_l0_reverse.copy_(torch.tensor(_ifog_to_torch(Ub, H)))
        lstm.bias_ih_l0_reverse.copy_(torch.tensor(_ifog_to_torch(bb, H))); lstm.bias_hh_l0_reverse.zero_()
    return lstm


def test_bilstmchar_equals_torch():
    """M9 == torch: nn.LSTM(bidirectional) over each rare word's characters, its final states h_n
    (forward after the last char, backward after the first) as the word vector, then M2 as nn.LSTM +
    Linear/tanh/Linear + cross-entropy; gradients by autograd (pins R-38's wiring: which final state,
    which half of the word vector, C_emb accumulation over repeated characters)."""
    H, E, C, V, Mh, Ec, Vc = 3, 4, 5, 6, 7, 3, 4
    P = _params("bilstmchar", H, E, C, 11, Mh, Ec=Ec, Vc=Vc)
    rng = np.random.default_rng(12)
    X = rng.uniform(-1, 1, (V, E))
    nodes = [((), 0, 1, ()), ((0,), 4, 2, (1, 3, 1, 0)), ((1,), 2, -1, ()), ((2,), 5, 0, (2,)),
             ((3,), 3, 4, ())]
    loss, G, dX = M.forward_backward("bilstmchar", P, X, [nodes], H)
    Hc = E // 2
    clstm = _torch_bilstm(P["Wcf"], P["Ucf"], P["bcf"], P["Wcb"], P["Ucb"], P["bcb"], Hc)
    wlstm = _torch_bilstm(P["Wf"], P["Uf"], P["bf"], P["Wb"], P["Ub"], P["bb"], H)
    mlp = torch.nn.Linear(2 * H, Mh, dtype=torch.float64)
    tag = torch.nn.Linear(Mh, C, dtype=torch.float64)
    with torch.no_grad():
        mlp.weight.copy_(torch.tensor(P["W_mlp"])); mlp.bias.copy_(torch.tensor(P["b_mlp"]))
        tag.weight.copy_(torch.tensor(P["W_tag"])); tag.bias.copy_(torch.tensor(P["b_tag"]))
    cemb = torch.tensor(P["C_emb"], requires_grad=True)
    Xt = torch.tensor(X, requires_grad=True)
    rows = []
    for (_, tok, _, chars) in nodes:
        if chars:
            _, (hn, _) = clstm(cemb[list(chars)][:, None, :])
            rows.append(torch.cat([hn[0, 0], hn[1, 0]]))
        else:
            rows.append(Xt[tok])
    out, _ = wlstm(torch.stack(rows)[:, None, :])
    z = tag(torch.tanh(mlp(out[:, 0, :])))
    keep = [t for t, nd in enumerate(nodes) if nd[2] >= 0]
    lt = torch.nn.functional.cross_entropy(z[keep], torch.tensor([nodes[t][2] for t in keep]), reduction="sum")
    lt.backward()
    assert abs(loss - lt.item()) < 1e-12
    np.testing.assert_allclose(G["C_emb"], cemb.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(dX, Xt.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(_ifog_to_torch(G["Wcf"], Hc), clstm.weight_ih_l0.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(_ifog_to_torch(G["Ucb"], Hc), clstm.weight_hh_l0_reverse.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(_ifog_to_torch(G["bcb"], Hc), clstm.bias_ih_l0_reverse.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(_ifog_to_torch(G["Wb"], H), wlstm.weight_ih_l0_reverse.grad.numpy(), atol=1e-12)


def test_bilstmchar_without_rare_words_is_bilstm():
    """Special case: with no spelled word M9 is M2 exactly, and the character parameters get zero gradient."""
    H, E, C, V = 4, 6, 5, 9
    P = _params("bilstmchar", H, E, C, 13, 5, Ec=3, Vc=5)
    rng = np.random.default_rng(14)
    X = rng.uniform(-1, 1, (V, E))
    graphs = synth.tagger_batch(rng, 3, (2, 6), V, C)
    l9, G9, dX9 = M.forward_backward("bilstmchar", P, X, [[nd + ((),) for nd in g] for g in graphs], H)
    P2 = {k: P[k] for k, _ in M.param_shapes("bilstm", H, E, C, 5)}
    l2, G2, dX2 = M.forward_backward("bilstm", P2, X, graphs, H)
    assert l9 == l2
    for k in P2:
        np.testing.assert_array_equal(G9[k], G2[k])
    np.testing.assert_array_equal(dX9, dX2)
    for k in ("C_emb", "Wcf", "Ucf", "Wcb", "Ucb", "bcf", "bcb"):
        assert not G9[k].any()


def test_bilstmchar_synthetic_batch():
    """Input recipe (R-38): spellings are a function of the word id; validation accepts the batch and
    rejects spellings outside the character set or on another cell."""
    g = synth.config_batch("bilstmchar", 0, batch=32)
    spelled = {}
    for nodes in g:
        for nd in nodes:
            if nd[3]:
                assert spelled.setdefault(nd[1], nd[3]) == nd[3]
                assert 2 <= len(nd[3]) <= 12
    assert spelled
    M.validate("bilstmchar", g, 4096, 9, n_chars=64)
    with pytest.raises(ValueError):
        M.validate("bilstmchar", g, 4096, 9, n_chars=8 if max(max(s) for s in spelled.values()) >= 8 else 0)
    with pytest.raises(ValueError):
        M.validate("bilstm", g, 4096, 9, n_chars=64)


def test_fd_tdlstm():
    rng = np.random.default_rng(15)
    _fd_check("tdlstm", [synth.td_pyramid(rng, 3, 3, 3), synth.td_pyramid(rng, 2, 3, 3)], H=2, E=2, C=3, V=3)


def test_gru_equals_torch_grucell():
    """M5 (reading R-34) == torch.nn.GRUCell in float64: torch stacks (r, z, n) in weight_ih / weight_hh
    with separate biases and applies the reset gate to W_hn h + b_hn, as the oracle does — a swapped gate,
    a reset applied before U_n, or a wrong sign of the (1 - z) / z interpolation fails this."""
    H, E, C, V = 5, 4, 6, 7
    P = _params("gru", H, E, C, 3)
    P = {k: v * 2.0 for k, v in P.items()}
    rng = np.random.default_rng(4)
    X = rng.uniform(-1, 1, (V, E))
    nodes = synth.chain(rng, 6, V, lm=True)
    loss, G, dX = M.forward_backward("gru", P, X, [nodes], H)
    cell = torch.nn.GRUCell(E, H, dtype=torch.float64)
    with torch.no_grad():
        cell.weight_ih.copy_(torch.tensor(P["W"])); cell.weight_hh.copy_(torch.tensor(P["U"]))
        cell.bias_ih.copy_(torch.tensor(P["b_i"])); cell.bias_hh.copy_(torch.tensor(P["b_h"]))
    Wo = torch.tensor(P["W_out"], requires_grad=True)
    bo = torch.tensor(P["b_out"], requires_grad=True)
    toks = [t for (_, t, _) in nodes]
    Xt = torch.tensor(np.array([X[t] for t in toks]), requires_grad=True)
    h = torch.zeros(1, H, dtype=torch.float64)
    ref = torch.zeros((), dtype=torch.float64)
    for t, (_, _, lab) in enumerate(nodes):
        h = cell(Xt[t:t + 1], h)
        if lab >= 0:
            ref = ref + torch.nn.functional.cross_entropy((h[0] @ Wo.T + bo)[None], torch.tensor([lab]),
                                                          reduction="sum")
    ref.backward()
    assert abs(loss - ref.item()) < 1e-12
    np.testing.assert_allclose(G["W"], cell.weight_ih.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["U"], cell.weight_hh.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["b_i"], cell.bias_ih.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["b_h"], cell.bias_hh.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["W_out"], Wo.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["b_out"], bo.grad.numpy(), atol=1e-12)
    dXref = np.zeros_like(X)
    for t, tok in enumerate(toks):
        dXref[tok] += Xt.grad.numpy()[t]
    np.testing.assert_allclose(dX, dXref, atol=1e-12)


def _torch_lstm_chain(Wih, Whh, b, xs, Wout, bout, labels):
    """Reference with torch.nn.LSTMCell (gate order i, f, g, o) + cross_entropy(sum)."""
    H = Whh.shape[1]
    cell = torch.nn.LSTMCell(Wih.shape[1], H, dtype=torch.float64)
    with torch.no_grad():
        cell.weight_ih.copy_(torch.tensor(Wih)); cell.weight_hh.copy_(torch.tensor(Whh))
        cell.bias_ih.copy_(torch.tensor(b)); cell.bias_hh.zero_()
    Wo = torch.tensor(Wout, requires_grad=True)
    bo = torch.tensor(bout, requires_grad=True)
    X = torch.tensor(np.array(xs), requires_grad=True)
    h = torch.zeros(1, H, dtype=torch.float64); c = torch.zeros(1, H, dtype=torch.float64)
    loss = torch.zeros((), dtype=torch.float64)
    for t in range(len(xs)):
        h, c = cell(X[t:t + 1], (h, c))
        if labels[t] >= 0:
            z = h[0] @ Wo.T + bo
            loss = loss + torch.nn.functional.cross_entropy(z[None], torch.tensor([labels[t]]), reduction="sum")
    loss.backward()
    return (loss.item(), cell.weight_ih.grad.numpy(), cell.weight_hh.grad.numpy(), cell.bias_ih.grad.numpy(),
            Wo.grad.numpy(), bo.grad.numpy(), X.grad.numpy())


def _ifog_to_torch(A, H):
    """oracle gate order (i, f, o, g) -> torch (i, f, g, o)."""
    return np.concatenate([A[0:H], A[H:2 * H], A[3 * H:4 * H], A[2 * H:3 * H]])


def test_lstm_equals_torch_lstmcell():
    H, E, C, V = 5, 4, 6, 7
    P = _params("lstm", H, E, C, 3)
    rng = np.random.default_rng(4)
    X = rng.uniform(-1, 1, (V, E))
    nodes = synth.chain(rng, 6, V, lm=True)
    loss, G, dX = M.forward_backward("lstm", P, X, [nodes], H)
    toks = [t for (_, t, _) in nodes]
    labs = [l for (_, _, l) in nodes]
    ref = _torch_lstm_chain(_ifog_to_torch(P["W"], H), _ifog_to_torch(P["U"], H), _ifog_to_torch(P["b"], H),
                            [X[t] for t in toks], P["W_out"], P["b_out"], labs)
    assert abs(loss - ref[0]) < 1e-12
    np.testing.assert_allclose(_ifog_to_torch(G["W"], H), ref[1], atol=1e-12)
    np.testing.assert_allclose(_ifog_to_torch(G["U"], H), ref[2], atol=1e-12)
    np.testing.assert_allclose(_ifog_to_torch(G["b"], H), ref[3], atol=1e-12)
    np.testing.assert_allclose(G["W_out"], ref[4], atol=1e-12)
    np.testing.assert_allclose(G["b_out"], ref[5], atol=1e-12)
    dXref = np.zeros_like(X)
    for t, tok in enumerate(toks):
        dXref[tok] += ref[6][t]
    np.testing.assert_allclose(dX, dXref, atol=1e-12)


@pytest.mark.parametrize("side", ["left", "right"])
def test_binary_comb_equals_torch_lstmcell(side):
    """M4 on a comb whose side leaves have zero embeddings (h = c = 0 there, since b_u = 0)
    is an LSTM chain over the spine with zero inputs after step 0 (see module docstring)."""
    H, E, C, T = 4, 3, 5, 5
    rng = np.random.default_rng(7)
    Wl = synth.init_params([("Wih", (4 * H, E)), ("Whh", (4 * H, H)), ("b", (4 * H,)), ("Wo", (C, H)),
                            ("bo", (C,))], rng)
    Wl["b"][2 * H:3 * H] = 0.0          # torch order i,f,g,o: b_g = 0 -> side leaves have u = 0
    Wi, Wf, Wg, Wo_ = (Wl["Wih"][k * H:(k + 1) * H] for k in range(4))
    Ui, Uf, Ug, Uo = (Wl["Whh"][k * H:(k + 1) * H] for k in range(4))
    bi, bf, bg, bo = (Wl["b"][k * H:(k + 1) * H] for k in range(4))
    Z = np.zeros((H, H))
    spine = np.concatenate([Ui, Uo, Ug])
    P = {"W_iou": np.concatenate([Wi, Wo_, Wg]),
         "U_iou": np.concatenate([spine, np.zeros((3 * H, H))], 1) if side == "left"
         else np.concatenate([np.zeros((3 * H, H)), spine], 1),
         "U_fl": Uf if side == "left" else Z, "U_fr": Z if side == "left" else Uf,
         "W_out": Wl["Wo"], "b_iou": np.concatenate([bi, bo, bg]), "b_f": bf, "b_out": Wl["bo"]}
    X = rng.uniform(-1, 1, (2, E)); X[1] = 0.0      # token 1 = the zero embedding
    nodes = [((), 0, -1)]
    spine_idx = 0
    for t in range(1, T):
        nodes.append(((), 1, -1))
        ch = (spine_idx, len(nodes) - 1) if side == "left" else (len(nodes) - 1, spine_idx)
        nodes.append((ch, -1, 2 if t == T - 1 else -1))
        spine_idx = len(nodes) - 1
    loss, G, dX = M.forward_backward("binary", P, X, [nodes], H)
    xs = [X[0]] + [np.zeros(E)] * (T - 1)
    ref = _torch_lstm_chain(Wl["Wih"], Wl["Whh"], Wl["b"], xs, Wl["Wo"], Wl["bo"], [-1] * (T - 1) + [2])
    assert abs(loss - ref[0]) < 1e-12
    dWih, dWhh = ref[1], ref[2]
    np.testing.assert_allclose(G["W_iou"], np.concatenate([dWih[0:H], dWih[3 * H:], dWih[2 * H:3 * H]]), atol=1e-12)
    half = G["U_iou"][:, :H] if side == "left" else G["U_iou"][:, H:]
    np.testing.assert_allclose(half, np.concatenate([dWhh[0:H], dWhh[3 * H:], dWhh[2 * H:3 * H]]), atol=1e-12)
    np.testing.assert_allclose(G["U_fl"] if side == "left" else G["U_fr"], dWhh[H:2 * H], atol=1e-12)
    np.testing.assert_allclose(G["b_f"], ref[3][H:2 * H], atol=1e-12)
    np.testing.assert_allclose(G["W_out"], ref[4], atol=1e-12)
    np.testing.assert_allclose(dX[0], ref[6][0], atol=1e-12)


def test_bilstm_equals_torch_lstm():
    H, E, C, V, Mh = 3, 4, 5, 6, 7
    P = _params("bilstm", H, E, C, 5, Mh)
    rng = np.random.default_rng(6)
    X = rng.uniform(-1, 1, (V, E))
    nodes = synth.chain(rng, 5, V, lm=False, n_tags=C)
    nodes[2] = (nodes[2][0], nodes[2][1], -1)
    loss, G, dX = M.forward_backward("bilstm", P, X, [nodes], H)
    lstm = torch.nn.LSTM(E, H, bidirectional=True, dtype=torch.float64)
    with torch.no_grad():
        lstm.weight_ih_l0.copy_(torch.tensor(_ifog_to_torch(P["Wf"], H)))
        lstm.weight_hh_l0.copy_(torch.tensor(_ifog_to_torch(P["Uf"], H)))
        lstm.bias_ih_l0.copy_(torch.tensor(_ifog_to_torch(P["bf"], H))); lstm.bias_hh_l0.zero_()
        lstm.weight_ih_l0_reverse.copy_(torch.tensor(_ifog_to_torch(P["Wb"], H)))
        lstm.weight_hh_l0_reverse.copy_(torch.tensor(_ifog_to_torch(P["Ub"], H)))
        lstm.bias_ih_l0_reverse.copy_(torch.tensor(_ifog_to_torch(P["bb"], H))); lstm.bias_hh_l0_reverse.zero_()
    mlp = torch.nn.Linear(2 * H, Mh, dtype=torch.float64)
    tag = torch.nn.Linear(Mh, C, dtype=torch.float64)
    with torch.no_grad():
        mlp.weight.copy_(torch.tensor(P["W_mlp"])); mlp.bias.copy_(torch.tensor(P["b_mlp"]))
        tag.weight.copy_(torch.tensor(P["W_tag"])); tag.bias.copy_(torch.tensor(P["b_tag"]))
    toks = [t for (_, t, _) in nodes]
    labs = [l for (_, _, l) in nodes]
    xs = torch.tensor(X[toks], requires_grad=True)
    out, _ = lstm(xs[:, None, :])
    z = tag(torch.tanh(mlp(out[:, 0, :])))
    keep = [t for t in range(len(labs)) if labs[t] >= 0]
    lt = torch.nn.functional.cross_entropy(z[keep], torch.tensor([labs[t] for t in keep]), reduction="sum")
    lt.backward()
    assert abs(loss - lt.item()) < 1e-12
    np.testing.assert_allclose(_ifog_to_torch(G["Wf"], H), lstm.weight_ih_l0.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(_ifog_to_torch(G["Ub"], H), lstm.weight_hh_l0_reverse.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["W_mlp"], mlp.weight.grad.numpy(), atol=1e-12)
    np.testing.assert_allclose(G["b_tag"], tag.bias.grad.numpy(), atol=1e-12)
    dXref = np.zeros_like(X)
    for t, tok in enumerate(toks):
        dXref[tok] += xs.grad.numpy()[t]
    np.testing.assert_allclose(dX, dXref, atol=1e-12)


def test_childsum_chain_equals_lstm():
    """SURVEY §8(c) invariant: M3 on a chain == M1 with W = [W_i; W_f; W_o; W_u] (same U, b)."""
    H, E, C, V = 4, 3, 5, 6
    P3 = _params("childsum", H, E, C, 8)
    rng = np.random.default_rng(9)
    X = rng.uniform(-1, 1, (V, E))
    nodes = synth.chain(rng, 7, C, lm=True)
    sl = lambda A, k: A[k * H:(k + 1) * H]
    P1 = {"W": np.concatenate([sl(P3["W_iou"], 0), P3["W_f"], sl(P3["W_iou"], 1), sl(P3["W_iou"], 2)]),
          "U": np.concatenate([sl(P3["U_iou"], 0), P3["U_f"], sl(P3["U_iou"], 1), sl(P3["U_iou"], 2)]),
          "b": np.concatenate([sl(P3["b_iou"], 0), P3["b_f"], sl(P3["b_iou"], 1), sl(P3["b_iou"], 2)]),
          "W_out": P3["W_out"], "b_out": P3["b_out"]}
    l3, G3, dX3 = M.forward_backward("childsum", P3, X, [nodes], H)
    l1, G1, dX1 = M.forward_backward("lstm", P1, X, [nodes], H)
    assert abs(l3 - l1) < 1e-12
    np.testing.assert_allclose(G3["W_f"], G1["W"][H:2 * H], atol=1e-12)
    np.testing.assert_allclose(G3["U_iou"], np.concatenate([G1["U"][0:H], G1["U"][2 * H:]]), atol=1e-12)
    np.testing.assert_allclose(G3["b_iou"], np.concatenate([G1["b"][0:H], G1["b"][2 * H:]]), atol=1e-12)
    np.testing.assert_allclose(dX3, dX1, atol=1e-12)


@pytest.mark.parametrize("cell", ["binary", "childsum", "lstm", "gru", "rvnn"])
def test_batch_order_and_linearity(cell):
    H, E, C, V = 4, 4, 5, 50
    P = _params(cell, H, E, C, 10)
    rng = np.random.default_rng(11)
    X = rng.uniform(-1, 1, (V, E))
    if cell in ("lstm", "gru"):
        graphs = [synth.chain(rng, int(rng.integers(2, 6)), C) for _ in range(4)]
    else:
        graphs = synth.tree_batch(rng, 4, (2, 7), V, C)
    l, G, dX = M.forward_backward(cell, P, X, graphs, H)
    lp, Gp, dXp = M.forward_backward(cell, P, X, graphs[::-1], H)
    assert abs(l - lp) < 1e-10
    for k in G:
        np.testing.assert_allclose(G[k], Gp[k], atol=1e-12)
    l1, G1, _ = M.forward_backward(cell, P, X, graphs[:1], H)
    l2, G2, _ = M.forward_backward(cell, P, X, graphs[:1] * 2, H)
    assert abs(l2 - 2 * l1) < 1e-12
    for k in G1:
        np.testing.assert_allclose(G2[k], 2 * G1[k], atol=1e-12)


def test_single_leaf_closed_form():
    H, E, C = 3, 2, 4
    P = _params("binary", H, E, C, 12)
    x = np.array([0.3, -0.7])
    a = P["W_iou"] @ x + P["b_iou"]
    s = lambda v: 1 / (1 + math.e ** (-v))
    h = [s(a[H + k]) * math.tanh(s(a[k]) * math.tanh(a[2 * H + k])) for k in range(H)]
    z = P["W_out"] @ np.array(h) + P["b_out"]
    expect = -(z[1] - math.log(sum(math.exp(v) for v in z)))
    loss, G, _ = M.forward_backward("binary", P, x[None, :], [[((), 0, 1)]], H)
    assert abs(loss - expect) < 1e-12
    # head closed form: dz = softmax(z) - onehot(y)  ->  db_out
    p = np.exp(z - z.max()); p /= p.sum(); p[1] -= 1
    np.testing.assert_allclose(G["b_out"], p, atol=1e-12)


def test_sgd_weight_decay():
    P = {"a": np.array([1.0, -2.0])}
    G = {"a": np.array([0.5, 0.25])}
    out = M.sgd(P, G, lr=0.1, weight_decay=0.01)
    np.testing.assert_allclose(out["a"], [1.0 - 0.1 * (0.5 + 0.01), -2.0 - 0.1 * (0.25 - 0.02)])


def test_table1_weights_once_bytes():
    """Tab.I VPPS row == (matrix floats of M4 at H=E=256, C=5) x 4 B x 128/batch, in MiB,
    truncated to 2 decimals."""
    mats = [s for (_, s) in M.param_shapes("binary", 256, 256, 5) if len(s) == 2]
    floats = sum(r * c for r, c in mats)
    assert floats == 11 * 256 * 256 + 5 * 256 == 722176
    rows = [l.split() for l in open(os.path.join(GOLD, "tab1_vpps_mb.txt")) if l.strip() and l[0] != "#"]
    for b, mb in rows:
        val = floats * 4 * (128 // int(b)) / 2 ** 20
        assert math.floor(val * 100) / 100 == float(mb), (b, val, mb)
    # the alternatives of SURVEY Appendix A miss the table (child-sum, 2-class head, N-ary with cross terms)
    alt_cs = sum(r * c for (_, s) in M.param_shapes("childsum", 256, 256, 5) if len(s) == 2 for r, c in [s])
    assert math.floor(alt_cs * 4 * 128 / 2 ** 20 * 100) / 100 != 352.62


def test_flop_count_units():
    """internal node 48H^2 FLOP, leaf 18HE with dX, root head 6CH."""
    H = E = 256
    assert M.flop_count("binary", [[((), 0, -1)]], H, E, 5) == 18 * H * E
    assert M.flop_count("binary", [[((), 0, -1), ((), 0, -1), ((0, 1), -1, 0)]], H, E, 5) == \
        2 * 18 * H * E + 48 * H * H + 6 * 5 * H


def test_validate_rules():
    with pytest.raises(ValueError):
        M.validate("binary", [[((), 0, -1), ((0,), -1, 1)]], 5, 5)     # unary internal node (R-26)
    with pytest.raises(ValueError):
        M.validate("binary", [[((), -1, 1)]], 5, 5)                     # leaf without a word
    M.validate("childsum", [[((), -1, -1), ((0,), 2, 1)]], 5, 5)


def _torch_chain_flops(P, xs, H, fwd_only_dir=False):
    """FLOPs that torch.utils.flop_counter counts for forward + backward of the M1/M2 definitions written
    with plain linear maps (the first step of a direction has no recurrent product: h_0 = 0)."""
    import torch
    from torch.utils.flop_counter import FlopCounterMode
    T = {k: torch.tensor(v, requires_grad=True) for k, v in P.items()}
    x = torch.tensor(np.stack(xs), requires_grad=True)
    lin = torch.nn.functional.linear

    def run(W, U, b, order):
        h = c = None
        out = {}
        for t in order:
            a = lin(x[t], W, b) if h is None else lin(x[t], W, b) + lin(h, U)
            i, f, o, g = torch.sigmoid(a[:H]), torch.sigmoid(a[H:2 * H]), torch.sigmoid(a[2 * H:3 * H]), torch.tanh(a[3 * H:])
            c = i * g if c is None else f * c + i * g
            h = o * torch.tanh(c)
            out[t] = h
        return out
    return T, x, run, lin, FlopCounterMode


def test_flop_count_bilstm_equals_torch_flop_counter():
    """flop_count('bilstm') (M2, L265/L281) against torch's own FLOP counter over forward + backward of the
    tagger written with plain linear maps: 2 FLOP per MAC for the forward product, dW and dx / dh."""
    import torch
    H, E, C, Mh = 3, 4, 5, 6
    P = _params("bilstm", H, E, C, 21, Mh)
    rng = np.random.default_rng(22)
    for n, labels in ((5, [1, -1, 2, 0, -1]), (1, [3]), (4, [-1, -1, -1, 1])):
        xs = [rng.standard_normal(E) for _ in range(n)]
        T, x, run, lin, FC = _torch_chain_flops(P, xs, H)
        with FC(display=False) as fc:
            hf = run(T["Wf"], T["Uf"], T["bf"], range(n))
            hb = run(T["Wb"], T["Ub"], T["bb"], range(n - 1, -1, -1))
            loss = 0
            for t, y in enumerate(labels):
                if y < 0:
                    continue
                m = torch.tanh(lin(torch.cat([hf[t], hb[t]]), T["W_mlp"], T["b_mlp"]))
                z = lin(m, T["W_tag"], T["b_tag"])
                loss = loss + torch.nn.functional.cross_entropy(z[None], torch.tensor([y]))
            # every position runs its backward step (as in the oracle and the device), also a trailing
            # unlabelled one whose gradient is zero: tie all states into the loss with weight 0
            loss = loss + 0 * sum(h.sum() for h in list(hf.values()) + list(hb.values()))
            loss.backward()
        nodes = [((t - 1,) if t else (), 0, y) for t, y in enumerate(labels)]
        assert M.flop_count("bilstm", [nodes], H, E, C, M=Mh) == fc.get_total_flops()
    assert M.flop_count("bilstm", [], H, E, C, M=Mh) == 0


def test_flop_count_lstm_equals_torch_flop_counter():
    import torch
    H, E, C = 3, 4, 5
    P = _params("lstm", H, E, C, 23)
    rng = np.random.default_rng(24)
    labels = [2, -1, 4, 0]
    xs = [rng.standard_normal(E) for _ in labels]
    T, x, run, lin, FC = _torch_chain_flops(P, xs, H)
    with FC(display=False) as fc:
        hs = run(T["W"], T["U"], T["b"], range(len(labels)))
        loss = sum(torch.nn.functional.cross_entropy(lin(hs[t], T["W_out"], T["b_out"])[None], torch.tensor([y]))
                   for t, y in enumerate(labels) if y >= 0)
        loss.backward()
    nodes = [((t - 1,) if t else (), 0, y) for t, y in enumerate(labels)]
    assert M.flop_count("lstm", [nodes], H, E, C) == fc.get_total_flops()


def test_full_size_golden_regenerates():
    """tests/golden/full_c3.npz is what tools/make_golden.py (oracle/ + synth/ only) writes: recompute the
    config-3 case (64 sentences, H = 256, V = 1000) and compare every stored value bit for bit."""
    import importlib.util
    import os
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    spec = importlib.util.spec_from_file_location("make_golden", os.path.join(root, "tools", "make_golden.py"))
    mg = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mg)
    g = np.load(os.path.join(root, "tests", "golden", "full_c3.npz"))
    graphs, P, X = mg.inputs("c3")
    loss, G, dX = M.forward_backward("lstm", P, X, graphs, 256)
    assert abs(loss - float(g["loss"])) <= 1e-9 * abs(loss)
    for k in G:
        flat = G[k].ravel()
        np.testing.assert_allclose(flat[g[f"{k}__idx"]], g[f"{k}__val"], rtol=1e-9, atol=1e-12)
        assert abs(np.abs(flat).max() - float(g[f"{k}__max"])) <= 1e-9 * float(g[f"{k}__max"])
    np.testing.assert_allclose(dX.ravel()[g["dX__idx"]], g["dX__val"], rtol=1e-9, atol=1e-12)
