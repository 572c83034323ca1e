"""GPU parity: the CUDA path (through the C ABI) against the FP64 oracle on the same seeded inputs.

Tolerance (BASELINE.json north_star; reading R-22): per tensor ‖g − o‖∞ / ‖o‖∞ ≤ 1e-4,
loss |L − L_o| / |L_o| ≤ 1e-4.  FP32 accumulation order differs (atomics), so bitwise equality is
not expected for floats; the integer artefacts are checked bit-exactly in test_host_parity.py.
"""
import numpy as np
import pytest

import synth
from oracle import models as M

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
TOL = 1e-4


def _vpps():
    from paper_conf_micro_khorasanieas18_b200 import vpps
    return vpps


def run_case(cell, H, E, C, graphs, V, seed=0, want_dx=True, sgd=None, groups=1, cluster=0, dataflow=False, level=0,
             mlp=256):
    vpps = _vpps()
    rng = np.random.default_rng(seed)
    shapes = vpps.param_shapes(cell, H, E, C, mlp)
    P = synth.init_params(shapes, rng)
    X = synth.input_table(rng, V, E)
    m = vpps.Model(cell, H, E, C, device=0, groups=groups, cluster=cluster, dataflow=dataflow, level=level, mlp=mlp)
    dev = torch.device("cuda:0")
    params = torch.zeros(m.n_floats, dtype=torch.float32, device=dev)
    grads = torch.full_like(params, float("nan"))
    views = m.views(params)
    for name, _ in shapes:
        views[name].copy_(torch.from_numpy(P[name]).float())
    m.bind(params, grads)
    inputs = torch.from_numpy(X).float().to(dev)
    dX = torch.full_like(inputs, float("nan")) if want_dx else None
    s = m.build_script(graphs)
    if sgd is None:
        m.fwd_bwd(s, inputs, dX)
    else:
        m.fwd_bwd_sgd(s, inputs, dX, lr=sgd[0], weight_decay=sgd[1])
    loss = m.latest_loss()
    torch.cuda.synchronize()
    return m, P, X, loss, params, grads, dX


def rel(a, b):
    return float(np.abs(np.asarray(a, np.float64) - b).max() / max(np.abs(b).max(), 1e-30))


_STATS = []


def elementwise(name, a, b):
    """R-22's elementwise statistics: |g - o| / max(|o|, 1e-3 ‖o‖∞) per element (max, 99.9th percentile),
    recorded for the report (VPPS_PARITY_STATS=path writes them as JSON lines at the end of the session)."""
    a = np.asarray(a, np.float64).ravel()
    b = np.asarray(b, np.float64).ravel()
    if b.size == 0:
        return
    floor = 1e-3 * max(np.abs(b).max(), 1e-30)
    r = np.abs(a - b) / np.maximum(np.abs(b), floor)
    _STATS.append(dict(tensor=name, max=float(r.max()), p999=float(np.quantile(r, 0.999)), n=int(b.size)))


@pytest.fixture(scope="session", autouse=True)
def _write_stats():
    yield
    import json
    import os
    path = os.environ.get("VPPS_PARITY_STATS")
    if path and _STATS:
        with open(path, "w") as f:
            for row in _STATS:
                f.write(json.dumps(row) + "\n")


def check(cell, H, E, C, graphs, V, seed=0, want_dx=True, groups=1, cluster=0, dataflow=False, level=0, mlp=256):
    m, P, X, loss, params, grads, dX = run_case(cell, H, E, C, graphs, V, seed, want_dx, groups=groups,
                                                cluster=cluster, dataflow=dataflow, level=level, mlp=mlp)
    lo, Go, dXo = M.forward_backward(cell, P, X, graphs, H)
    assert abs(loss - lo) <= TOL * abs(lo), (loss, lo)
    gv = m.views(grads.cpu())
    for name, _ in m.shapes:
        assert rel(gv[name].numpy(), Go[name]) <= TOL, name
        elementwise(f"{cell} H{H} {name}", gv[name].numpy(), Go[name])
    if want_dx:
        assert rel(dX.cpu().numpy(), dXo) <= TOL, "dX"
        elementwise(f"{cell} H{H} dX", dX.cpu().numpy(), dXo)
    return loss, lo


def _trees(seed, batch, leaves, V, C):
    return synth.tree_batch(np.random.default_rng(seed), batch, leaves, V, C)


@pytest.mark.parametrize("H", [32, 128])
def test_binary_small(H):
    check("binary", H, H, 5, _trees(1, 5, (1, 12), 40, 5), 40)


def test_binary_target_config():
    """TGT: binary Tree-LSTM H = E = 256, batch 16 SST-shaped trees (5-50 leaves), 148 SMs."""
    graphs = synth.config_batch("tgt", 0)
    check("binary", 256, 256, 5, graphs, 4096, seed=3)


@pytest.mark.parametrize("groups", [2, 4])
def test_binary_target_replica_groups(groups):
    """SPEC P1 replica groups: nodes spread over G groups, gradients summed across groups in-kernel."""
    check("binary", 256, 256, 5, synth.config_batch("tgt", 3), 4096, seed=5, groups=groups)


@pytest.mark.parametrize("b", [0, 5])
def test_binary_target_cluster_replicas(b):
    """Cluster path: 16-CTA cluster replicas, whole trees per cluster, dW by the gradient GEMM (L185)."""
    check("binary", 256, 256, 5, synth.config_batch("tgt", b), 4096, seed=11 + b, cluster=16)


@pytest.mark.parametrize("b", [0, 5, 9])
def test_binary_target_dataflow_groups(b):
    """Dataflow path: 16-CTA groups of a cooperative launch, epoch-tagged slots instead of barriers."""
    check("binary", 256, 256, 5, synth.config_batch("tgt", b), 4096, seed=21 + b, cluster=16, dataflow=True)


@pytest.mark.parametrize("E,b", [(128, 0), (256, 5), (128, 11)])
def test_dataflow_groups_hidden_128(E, b):
    """Dataflow path at H = 128: groups of 8 CTAs (H / 16 units of 16), 16 groups; the leaf GEMM at E = 128
    (two K groups) or 256 (PAPER L241 / Fig.9: the hidden size sets the register partition)."""
    check("binary", 128, E, 5, synth.config_batch("tgt", b), 4096, seed=41 + b, cluster=8, dataflow=True)
    check("binary", 128, E, 5, [[((), 3, 2)]], 8, cluster=8, dataflow=True)               # one leaf


@pytest.mark.parametrize("cell,H", [("childsum", 128), ("binary", 64)])
def test_auto_replica_groups_grid(cell, H):
    """groups = -1 (automatic): the grid kernel with 4 replica groups, parity against the FP64 oracle."""
    graphs = synth.config_batch("c2", 2) if cell == "childsum" else _trees(9, 12, (2, 20), 4096, 5)
    check(cell, H, H, 5, graphs, 4096, seed=12, groups=-1)


def test_dataflow_degenerate_and_repeated_passes():
    check("binary", 256, 256, 5, [[((), 3, 2)]], 8, cluster=16, dataflow=True)           # one leaf
    check("binary", 256, 256, 5, _trees(12, 3, (1, 9), 30, 5), 30, cluster=16, dataflow=True, want_dx=False)
    t = [((), 0, 1), ((), 1, -1), ((0, 1), -1, 3), ((), 2, -1), ((2, 3), -1, 0)]           # inner labels
    check("binary", 256, 256, 5, [t, t], 4, cluster=16, dataflow=True)


def test_dataflow_epochs_across_passes():
    """Tagged slots are reused by later passes (and by other scripts) without clearing."""
    vpps = _vpps()
    rng = np.random.default_rng(31)
    H, C, V = 256, 5, 64
    shapes = vpps.param_shapes("binary", H, H, C)
    P = synth.init_params(shapes, rng)
    m = vpps.Model("binary", H, H, C, cluster=16, dataflow=True)
    params = torch.zeros(m.n_floats, device="cuda")
    grads = torch.zeros_like(params)
    for name, _ in shapes:
        m.views(params)[name].copy_(torch.from_numpy(P[name]).float())
    m.bind(params, grads)
    X = torch.from_numpy(synth.input_table(rng, V, H)).float().cuda()
    batches = [_trees(40 + i, 6, (2, 30), V, C) for i in range(3)]
    scripts = [m.build_script(b) for b in batches]
    for rep in range(2):
        for k, (b, s) in enumerate(zip(batches, scripts)):
            m.fwd_bwd(s, X)
            lo, Go, _ = M.forward_backward("binary", P, X.cpu().double().numpy(), b, H)
            loss = m.latest_loss()
            assert abs(loss - lo) <= TOL * abs(lo), (rep, k, loss, lo)
            gv = m.views(grads.cpu())
            for name, _ in m.shapes:
                assert rel(gv[name].numpy(), Go[name]) <= TOL, (rep, name)


def test_cluster_degenerate_batches():
    check("binary", 256, 256, 5, [[((), 3, 2)]], 8, cluster=16)              # one leaf: most clusters idle
    check("binary", 256, 256, 5, _trees(12, 3, (1, 9), 30, 5), 30, cluster=16, want_dx=False)


def check_update(m, P, Pn, params):
    """Updated parameters against the oracle's SGD step θ' = θ − η(g + λθ) (L129, L197): per tensor the
    step itself within 1e-4 relative (R-22), plus the one FP32 rounding of the stored parameter
    (2^-24 of |θ'|, the floor below which no FP32 update can be resolved)."""
    pv = m.views(params.cpu())
    for name, _ in m.shapes:
        got = pv[name].double().numpy()
        step = Pn[name] - P[name]
        bound = TOL * np.abs(step).max() + 2.0 ** -22 * np.abs(Pn[name]).max()
        assert np.abs(got - Pn[name]).max() <= bound, (name, np.abs(got - Pn[name]).max(), bound)


@pytest.mark.parametrize("groups,cluster,dataflow", [(1, 0, False), (2, 0, False), (4, 0, False), (1, 16, False),
                                                     (1, 16, True)])
def test_fused_sgd_target_groups(groups, cluster, dataflow):
    graphs = synth.config_batch("tgt", 4)
    lr, wd = 0.05, 1e-3
    m, P, X, loss, params, grads, dX = run_case("binary", 256, 256, 5, graphs, 4096, seed=6, sgd=(lr, wd),
                                                groups=groups, cluster=cluster, dataflow=dataflow)
    lo, Go, _ = M.forward_backward("binary", P, X, graphs, 256)
    assert abs(loss - lo) <= TOL * abs(lo)
    check_update(m, P, M.sgd(P, Go, lr, wd), params)


@pytest.mark.parametrize("E", [128, 256])
def test_fused_sgd_dataflow_hidden_128(E):
    """vpps_fwd_bwd_sgd on 8-CTA dataflow groups (H = 128): the updated parameters against the FP64 oracle's
    SGD step at 1e-4 of the step (+ two FP32 roundings)."""
    graphs = synth.config_batch("tgt", 6)
    lr, wd = 0.05, 1e-3
    m, P, X, loss, params, grads, dX = run_case("binary", 128, E, 5, graphs, 4096, seed=8, sgd=(lr, wd),
                                                cluster=8, dataflow=True)
    lo, Go, _ = M.forward_backward("binary", P, X, graphs, 128)
    assert abs(loss - lo) <= TOL * abs(lo)
    check_update(m, P, M.sgd(P, Go, lr, wd), params)


@pytest.mark.parametrize("cell,H,level", [("binary", 256, 0), ("binary", 256, 1), ("bilstm", 64, 0),
                                          ("gru", 64, 0), ("rvnn", 64, 0)])
def test_fwd_bwd_then_sgd_step(cell, H, level):
    """The data-parallel step's two calls on one GPU (north_star): vpps_fwd_bwd writes the
    gradient (checked at 1e-4), then vpps_sgd_step (the K3 sgd_kernel) applies θ − η(g + λθ); on the
    dataflow path (binary, level = 0: leaf GEMM + vpps_df + gradient GEMM without its fused SGD tail) and
    on level paths."""
    lr, wd = 0.05, 1e-3
    if cell == "binary":
        graphs, V, C, kw = synth.config_batch("tgt", 11), 4096, 5, dict(cluster=16, dataflow=True) if not level \
            else dict(level=1)
    elif cell == "rvnn":
        graphs, V, C, kw = _trees(13, 6, (1, 20), 64, 5), 64, 5, {}
    else:
        graphs, V, C, kw = synth.tagger_batch(np.random.default_rng(14), 5, (1, 12), 64, 9), 64, 9, \
            dict(mlp=32) if cell == "bilstm" else {}
    m, P, X, loss, params, grads, dX = run_case(cell, H, H, C, graphs, V, seed=15, **kw)
    lo, Go, dXo = M.forward_backward(cell, P, X, graphs, H)
    assert abs(loss - lo) <= TOL * abs(lo)
    gv = m.views(grads.cpu())
    for name, _ in m.shapes:
        assert rel(gv[name].numpy(), Go[name]) <= TOL, name
    m.sgd_step(lr, wd)
    torch.cuda.synchronize()
    check_update(m, P, M.sgd(P, Go, lr, wd), params)


@pytest.mark.parametrize("cell,H", [("binary", 64), ("rvnn", 64), ("bilstm", 32), ("gru", 32), ("tdlstm", 32)])
def test_level_paths_fused_sgd(cell, H):
    """vpps_fwd_bwd_sgd on the level-synchronous paths (the pass, then the SGD kernel on the same stream)."""
    lr, wd = 0.1, 1e-2
    if cell in ("binary", "rvnn"):
        graphs, V, C, kw = _trees(16, 5, (1, 15), 32, 5), 32, 5, dict(level=1) if cell == "binary" else {}
    elif cell == "tdlstm":
        rng = np.random.default_rng(17)
        graphs, V, C, kw = [synth.td_pyramid(rng, n, 16, 5) for n in (6, 1, 4)], 16, 5, {}
    else:
        graphs, V, C, kw = synth.tagger_batch(np.random.default_rng(18), 4, (1, 10), 32, 7), 32, 7, \
            dict(mlp=16) if cell == "bilstm" else {}
    m, P, X, loss, params, grads, dX = run_case(cell, H, H, C, graphs, V, seed=19, sgd=(lr, wd), **kw)
    lo, Go, _ = M.forward_backward(cell, P, X, graphs, H)
    assert abs(loss - lo) <= TOL * abs(lo)
    check_update(m, P, M.sgd(P, Go, lr, wd), params)


def test_binary_target_other_batches():
    for b in (1, 7):
        check("binary", 256, 256, 5, synth.config_batch("tgt", b), 4096, seed=b)


def test_binary_degenerate_single_leaf_and_no_dx():
    graphs = [[((), 3, 2)], [((), 1, 0)]]               # lone labelled leaves: one cell level + heads
    check("binary", 32, 32, 5, graphs, 8)
    check("binary", 32, 32, 5, _trees(4, 3, (2, 6), 8, 5), 8, want_dx=False)


def test_binary_labels_on_inner_nodes():
    t = [((), 0, 1), ((), 1, -1), ((0, 1), -1, 3), ((), 2, -1), ((2, 3), -1, 0)]
    check("binary", 32, 32, 5, [t, t], 4)


def test_childsum_config2():
    graphs = synth.config_batch("c2", 0)
    check("childsum", 128, 128, 5, graphs, 4096, seed=2)


def test_childsum_arity_and_missing_tokens():
    g = [((), -1, -1), ((0,), 3, 2), ((), 4, -1), ((), 5, -1), ((1, 2, 3), -1, 1), ((), 1, -1),
         ((4, 5), 2, 4)]
    check("childsum", 32, 32, 5, [g] + _trees(5, 2, (1, 7), 8, 5), 8)


@pytest.mark.parametrize("level", [0, 1])
def test_lstm_config1(level):
    """Config 1 on the default path (the one-kernel grid kernel at H = 32) and on the chain recurrence + dense
    products."""
    graphs = synth.config_batch("c1", 0)
    check("lstm", 32, 32, 16, graphs, 16, seed=1, level=level)


def test_lstm_h256_small_vocab():
    rng = np.random.default_rng(9)
    graphs = [synth.chain(rng, int(rng.integers(5, 30)), 16) for _ in range(4)]
    check("lstm", 256, 256, 16, graphs, 16, seed=9)
    check("lstm", 256, 256, 16, graphs, 16, seed=9, level=-1)


@pytest.mark.parametrize("batch", [1, 4, 16, 64])
def test_lstm_config3_batch_sweep(batch):
    """Config 3 (LSTM LM, H = E = 256, sentences of 5-60 tokens, batch 1/4/16/64) with the GPU reading of
    the vocabulary (R-31: V = C = 32 symbols, the head held in one CTA's shared memory)."""
    graphs = synth.config_batch("c3", 0, batch=batch, V=32, C=32)
    check("lstm", 256, 256, 32, graphs, 32, seed=30 + batch, level=-1)
    check("lstm", 256, 256, 32, graphs, 32, seed=30 + batch)


@pytest.mark.parametrize("cell,H,groups", [("lstm", 256, 2), ("childsum", 128, 2), ("childsum", 128, 4)])
def test_grid_replica_groups(cell, H, groups):
    """Replica groups (R-28) of the grid kernel for configs 2 and 3: nodes split over G groups by the
    min-load rule, gradients summed across groups in the epilogue."""
    if cell == "lstm":
        graphs = synth.config_batch("c3", 1, batch=16, V=32, C=32)
        check("lstm", H, H, 32, graphs, 32, seed=40 + groups, groups=groups, level=-1)
    else:
        check("childsum", H, H, 5, synth.config_batch("c2", 1), 4096, seed=50 + groups, groups=groups)


def test_level_path_target_batch():
    """Level-synchronous GEMM path (vpps_level.cu) on the target config's shapes (H = E = 256)."""
    check("binary", 256, 256, 5, synth.config_batch("tgt", 2), 4096, seed=61, level=1)


def test_level_path_degenerate():
    check("binary", 64, 64, 5, [[((), 3, 2)]], 8, level=1)                                # one labelled leaf
    check("binary", 64, 32, 7, _trees(5, 3, (1, 9), 30, 7), 30, level=1, want_dx=False)
    g = [((), 1, -1), ((), 0, -1), ((0, 1), -1, 3), ((), 2, -1), ((2, 3), -1, 1)]      # inner labels
    check("binary", 64, 64, 5, [g], 4, level=1)


def test_level_path_config5_small():
    """Config 5's cell size (binary Tree-LSTM H = E = 1024) on a few small trees: the level path is what
    define_model picks automatically when no register-resident specialisation exists."""
    graphs = synth.config_batch("c5", 0, batch=3, leaves=(3, 9))
    check("binary", 1024, 1024, 5, graphs, 4096, seed=62)


def test_level_path_config5_full_batch_additivity():
    """Config 5 at its full per-GPU size (64 SST-shaped trees, H = E = 1024), where the FP64 oracle is too
    slow: the summed loss and every gradient are additive over a split of the batch (SURVEY c.5 batch
    invariant, the property the DP all-reduce relies on), and the full batch's loss is finite."""
    vpps = _vpps()
    graphs = synth.config_batch("c5", 0)
    res = []
    for part in (graphs, graphs[:32], graphs[32:]):
        _, _, _, loss, params, grads, dX = run_case("binary", 1024, 1024, 5, part, 4096, seed=63)
        res.append((loss, grads.double().cpu().numpy(), dX.double().cpu().numpy()))
    (l0, g0, x0), (l1, g1, x1), (l2, g2, x2) = res
    assert np.isfinite(l0) and abs(l0 - (l1 + l2)) <= 1e-4 * abs(l0), (l0, l1 + l2)
    assert rel(g1 + g2, g0) <= 1e-4
    assert rel(x1 + x2, x0) <= 1e-4


def test_tagger_small():
    """BiLSTM tagger (M2, config 4's model) on the level path: small sizes, ragged sentence lengths."""
    rng = np.random.default_rng(70)
    graphs = synth.tagger_batch(rng, 3, (1, 8), 50, 9)
    check("bilstm", 32, 32, 9, graphs, 50, seed=71, mlp=16)


def test_tagger_empty_sentences_in_batch():
    """Edge case: empty sentences mixed into a batch (ragged down to length 0) change nothing."""
    rng = np.random.default_rng(74)
    graphs = synth.tagger_batch(rng, 2, (1, 6), 50, 9)
    check("bilstm", 32, 32, 9, [[]] + graphs[:1] + [[]] + graphs[1:], 50, seed=75, mlp=16)


def test_tagger_config4_shapes():
    """Config 4's sizes (H = E = 512, MLP 256, 9 tags) on a few short sentences."""
    graphs = synth.config_batch("c4", 0, batch=4, lengths=(3, 12))
    check("bilstm", 512, 512, 9, graphs, 4096, seed=72, mlp=256)


def test_tagger_config4_full_batch_additivity():
    """Config 4 at its full size (16 sentences of 5-60 tokens): loss and gradients additive over a split."""
    graphs = synth.config_batch("c4", 1)
    res = []
    for part in (graphs, graphs[:8], graphs[8:]):
        _, _, _, loss, params, grads, dX = run_case("bilstm", 512, 512, 9, part, 4096, seed=73, mlp=256)
        res.append((loss, grads.double().cpu().numpy(), dX.double().cpu().numpy()))
    (l0, g0, x0), (l1, g1, x1), (l2, g2, x2) = res
    assert np.isfinite(l0) and abs(l0 - (l1 + l2)) <= 1e-4 * abs(l0), (l0, l1 + l2)
    assert rel(g1 + g2, g0) <= 1e-4
    assert rel(x1 + x2, x0) <= 1e-4


@pytest.mark.parametrize("batch", [1, 4])
def test_lstm_lm_config3_vocab1000(batch):
    """Config 3 as BASELINE states it (LSTM LM H = 256, V = 1000 next-token head, R-25): the vocabulary head
    exceeds one CTA's shared memory, so define_model takes the level path (head as a dense product)."""
    graphs = synth.config_batch("c3", 2, batch=batch, lengths=(5, 20))
    check("lstm", 256, 256, 1000, graphs, 1000, seed=80 + batch)


def test_lstm_lm_config3_full_batch_additivity():
    graphs = synth.config_batch("c3", 3, batch=64)
    res = []
    for part in (graphs, graphs[:32], graphs[32:]):
        m, _, _, loss, params, grads, dX = run_case("lstm", 256, 256, 1000, part, 1000, seed=84)
        gv = m.views(grads.cpu())
        res.append((loss, np.concatenate([gv[n].double().numpy().ravel() for n, _ in m.shapes]), dX.double().cpu().numpy()))
    (l0, g0, x0), (l1, g1, x1), (l2, g2, x2) = res
    assert np.isfinite(l0) and abs(l0 - (l1 + l2)) <= 1e-4 * abs(l0), (l0, l1 + l2)
    assert rel(g1 + g2, g0) <= 1e-4
    assert rel(x1 + x2, x0) <= 1e-4


def test_fused_sgd_update():
    graphs = _trees(6, 4, (1, 9), 20, 5)
    lr, wd = 0.05, 1e-3
    m, P, X, loss, params, grads, dX = run_case("binary", 32, 32, 5, graphs, 20, seed=6, sgd=(lr, wd))
    lo, Go, _ = M.forward_backward("binary", P, X, graphs, 32)
    check_update(m, P, M.sgd(P, Go, lr, wd), params)


def test_dp_split_equals_union():
    """Data parallelism invariant on one GPU: Σ gradients of the shards == gradient of the union."""
    graphs = synth.config_batch("tgt", 2)

    def grads_of(gs):
        m, _, _, _, _, grads, _ = run_case("binary", 256, 256, 5, gs, 4096, seed=4)
        return {k: v.numpy() for k, v in m.views(grads.cpu()).items()}

    g_all, g_a, g_b = grads_of(graphs), grads_of(graphs[:7]), grads_of(graphs[7:])
    for k in g_all:
        assert rel(g_a[k] + g_b[k], g_all[k]) <= TOL, k


def test_stale_and_latest_loss():
    vpps = _vpps()
    rng = np.random.default_rng(7)
    H, C, V = 32, 5, 16
    shapes = vpps.param_shapes("binary", H, H, C)
    P = synth.init_params(shapes, rng)
    m = vpps.Model("binary", H, H, C)
    params = torch.zeros(m.n_floats, device="cuda")
    grads = torch.zeros_like(params)
    for name, _ in shapes:
        m.views(params)[name].copy_(torch.from_numpy(P[name]).float())
    m.bind(params, grads)
    X = torch.from_numpy(synth.input_table(rng, V, H)).float().cuda()
    batches = [_trees(10 + i, 3, (1, 6), V, C) for i in range(3)]
    losses = []
    for b in batches:
        m.fwd_bwd(m.build_script(b), X)
        losses.append(M.forward_backward("binary", P, X.cpu().double().numpy(), b, H)[0])
    stale = m.stale_loss()          # loss of batch 1 (the pass before the most recent)
    latest = m.latest_loss()        # loss of batch 2
    assert abs(stale - losses[1]) <= TOL * abs(losses[1])
    assert abs(latest - losses[2]) <= TOL * abs(losses[2])


def test_errors_are_loud():
    vpps = _vpps()
    with pytest.raises(vpps.VppsError):
        vpps.Model("binary", 4096, 4096, 5)               # NOFIT
    m = vpps.Model("binary", 32, 32, 5)
    s = m.build_script(_trees(1, 2, (1, 5), 8, 5))
    with pytest.raises(vpps.VppsError):                   # buffers not bound
        m.fwd_bwd(s, torch.zeros(8, 32, device="cuda"))


@pytest.mark.parametrize("env", ["VPPS_LEAF_TC", "VPPS_LEAF_TMA", "VPPS_DW_TC", "VPPS_DW_TC2"])
def test_tensor_core_variants_subprocess(env):
    """The dataflow path's opt-in kernels against the oracle: the tensor-core leaf GEMM, the tcgen05 variant
    of the per-group gradient-GEMM items (VPPS_DW_TC) and the gathered 128 x 128 tensor-core gradient GEMM
    of vpps_dwtc.cu (VPPS_DW_TC2).  The switches are read once per process, so each runs in a child process."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = ("import sys; sys.path.insert(0, %r); sys.path.insert(0, %r); import test_gpu_parity as t; "
            "t.check('binary', 256, 256, 5, t._trees(3, 16, (5, 50), 4096, 5), 4096, cluster=16, dataflow=True); "
            "print('ok')" % (root, os.path.join(root, "tests")))
    r = subprocess.run([sys.executable, "-c", code], env={**os.environ, **{e: "1" for e in env.split("+")}},
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0 and "ok" in r.stdout, r.stdout + r.stderr


def test_gru_small():
    """M5 GRU chains (reading R-34) on the level path, config-1 shapes (H = E = 32, 4 sequences of 2-5)."""
    graphs = synth.config_batch("c1", 1)
    check("gru", 32, 32, 16, graphs, 16, seed=41)


@pytest.mark.parametrize("batch", [1, 4, 16])
def test_gru_lm_h256_vocab1000(batch):
    """GRU language model at config-3 shapes (H = E = 256, V = C = 1000, sentences of 5-60 tokens)."""
    graphs = synth.config_batch("c3", 4, batch=batch, lengths=(5, 40))
    check("gru", 256, 256, 1000, graphs, 1000, seed=90 + batch)


def test_gru_degenerate_chains():
    """Single-token chains, unlabelled positions and a repeated token (dX accumulation)."""
    g1 = [([], 3, 2)]
    g2 = [([], 1, -1), ([0], 1, -1), ([1], 1, 4)]
    g3 = [([], 0, 1), ([0], 5, -1)]
    check("gru", 32, 32, 8, [g1, g2, g3], 8, seed=43)


def test_rvnn_small():
    """M6 RvNN (reading R-35, untied leaf / internal weights) on the level path, small trees."""
    check("rvnn", 32, 32, 5, _trees(61, 6, (1, 9), 16, 5), 16, seed=61)


@pytest.mark.parametrize("b", [0, 1])
def test_rvnn_paper_size(b):
    """RvNN at the paper's size (Fig. 12: hidden and embedding 512) on SST-shaped trees, batch 16."""
    check("rvnn", 512, 512, 5, synth.config_batch("tgt", 20 + b), 4096, seed=62 + b)


def test_rvnn_labels_on_inner_nodes_and_single_leaves():
    g1 = [([], 1, 2)]                                           # a single labelled leaf
    g2 = [([], 0, -1), ([], 3, 1), ([0, 1], -1, 4), ([], 3, -1), ([2, 3], -1, 0)]
    check("rvnn", 64, 64, 5, [g1, g2] + _trees(64, 3, (2, 12), 8, 5), 8, seed=64)


@pytest.mark.parametrize("batch", [1, 4, 64])
def test_dataflow_batch_sweep(batch):
    """The bench's path (dataflow groups) at batch 1 / 4 / 64 (BASELINE's TGT batch sweep): at 64 trees a
    group runs ~7 trees, so its program spans several shared-memory chunks (refills) and its slots regions
    are the largest the bench sees."""
    check("binary", 256, 256, 5, synth.config_batch("tgt", 40 + batch, batch=batch), 4096, seed=70 + batch,
          cluster=16, dataflow=True)


def test_tdrnn_small():
    """M7 TD-RNN (reading R-36): pyramids over sentences — every inner node below the top has two parents,
    so a level's backward scatters two dh contributions into one child; includes a one-token sentence."""
    rng = np.random.default_rng(71)
    graphs = [synth.td_pyramid(rng, n, 16, 5) for n in (7, 1, 4, 12, 2)]
    check("tdrnn", 32, 32, 5, graphs, 16, seed=71)


def test_tdrnn_paper_size():
    """TD-RNN at the paper's size (Fig. 12: hidden and embedding 512), SST-length sentences."""
    graphs = synth.td_batch(np.random.default_rng(72), 4, lengths=(5, 20), vocab=4096)
    check("tdrnn", 512, 512, 5, graphs, 4096, seed=72)


def test_tdlstm_small_and_paper_size():
    """M8 TD-LSTM (reading R-37): the binary Tree-LSTM cell on TD pyramids (shared children: dh and dc from
    two parents per level, accumulated atomically) — small shapes and the paper's H = E = 256."""
    rng = np.random.default_rng(81)
    check("tdlstm", 32, 32, 5, [synth.td_pyramid(rng, n, 16, 5) for n in (6, 1, 3, 9)], 16, seed=81)
    check("tdlstm", 256, 256, 5, synth.td_batch(np.random.default_rng(82), 4, lengths=(5, 20)), 4096, seed=82)


def test_tdrnn_config_batch():
    """TD-RNN at the sweep's full configuration (16 pyramids over sentences of 5-30 tokens, H = E = 512):
    the whole batch against the oracle."""
    check("tdrnn", 512, 512, 5, synth.config_batch("tdrnn", 3), 4096, seed=73)


def _golden(case):
    import os
    return np.load(os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", f"full_{case}.npz"))


@pytest.mark.parametrize("case,cell,H,C,V,mlp,cfg,b,batch,seed", [
    ("c5", "binary", 1024, 5, 4096, 256, "c5", 0, None, 63),
    ("c4", "bilstm", 512, 9, 4096, 256, "c4", 1, None, 73),
    ("c3", "lstm", 256, 1000, 1000, 256, "c3", 3, 64, 84)])
def test_full_size_against_oracle_golden(case, cell, H, C, V, mlp, cfg, b, batch, seed):
    """BASELINE.json configs 5, 4, 3 at their full sizes (64 trees at H = 1024; 16 sentences of 5-60 tokens
    at H = 512; 64 sentences at H = 256, V = 1000) in the configuration define_model picks, against the
    FP64 oracle: the loss, and 2048 sampled entries of every gradient and of dX (tests/golden/full_*.npz,
    written by tools/make_golden.py from oracle/ and synth/ only) within 1e-4 of the tensor's max |value|
    (R-22)."""
    g = _golden(case)
    graphs = synth.config_batch(cfg, b, batch=batch)
    m, P, X, loss, params, grads, dX = run_case(cell, H, H, C, graphs, V, seed=seed, mlp=mlp)
    assert abs(loss - float(g["loss"])) <= TOL * abs(float(g["loss"])), (loss, float(g["loss"]))
    gv = m.views(grads.cpu())
    for name, _ in m.shapes:
        flat = gv[name].double().numpy().ravel()
        idx, val, mx = g[f"{name}__idx"], g[f"{name}__val"], float(g[f"{name}__max"])
        assert np.abs(flat[idx] - val).max() <= TOL * mx, name
    dflat = dX.cpu().double().numpy().ravel()
    assert np.abs(dflat[g["dX__idx"]] - g["dX__val"]).max() <= TOL * float(g["dX__max"]), "dX"


@pytest.mark.parametrize("H,batch", [(64, 5), (128, 40), (256, 70)])
def test_chain_recurrence_hidden_sizes(H, batch):
    """The register-resident chain recurrence (vpps_chain.cu) at every hidden size it is built for, against the
    oracle: LSTM LM at V = C = 100 on ragged sentences (incl. length 1), and a batch larger than one group's
    16-sentence slice (several groups, several slices per step at H = 256 with 70 sentences)."""
    rng = np.random.default_rng(300 + H)
    graphs = [synth.chain(rng, int(rng.integers(1, 30)), 100, lm=True) for _ in range(batch)]
    check("lstm", H, H, 100, graphs, 100, seed=301 + H)


def test_chain_tagger_paths_agree_subprocess():
    """VPPS_CHAIN=0 (per-step products, the level path before the register-resident recurrence) still matches
    the oracle on the tagger (both directions)."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = ("import sys; sys.path.insert(0, %r); sys.path.insert(0, %r); import test_gpu_parity as t; "
            "t.test_tagger_small(); t.test_chain_recurrence_hidden_sizes(128, 40); print('ok')"
            % (root, os.path.join(root, "tests")))
    r = subprocess.run([sys.executable, "-c", code], env={**os.environ, "VPPS_CHAIN": "0"}, capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0 and "ok" in r.stdout, r.stdout + r.stderr


def test_autotune_on_device_then_parity():
    """vpps.autotune times every device path this build offers for an LSTM LM at H = 256, C = 32 (grid kernel
    at G = 1 / 2, chain recurrence, per-step products) on sample batches and keeps the fastest; the chosen
    path then matches the oracle."""
    vpps = _vpps()
    rng = np.random.default_rng(500)
    sample = [[synth.chain(rng, int(rng.integers(5, 40)), 32, lm=True) for _ in range(16)] for _ in range(2)]
    X = torch.from_numpy(synth.input_table(rng, 32, 256)).float().cuda()
    best, res = vpps.autotune("lstm", 256, 256, 32, sample, X)
    assert len(res) >= 3 and min(res.values()) == res[repr(best)]
    graphs = synth.config_batch("c3", 7, batch=16, V=32, C=32)
    check("lstm", 256, 256, 32, graphs, 32, seed=501, groups=best.get("groups", 1), level=best.get("level", 0))


def _char_check(H, E, graphs, V, seed, mlp, C=9):
    """BiLSTMwChar through the C ABI against the oracle M9 (loss, every gradient incl. C_emb and the character
    LSTMs, and dX; rare words' table rows get no gradient)."""
    vpps = _vpps()
    rng = np.random.default_rng(seed)
    shapes = vpps.param_shapes("bilstmchar", H, E, C, mlp)
    P = synth.init_params(shapes, rng)
    X = synth.input_table(rng, V, E)
    m = vpps.Model("bilstmchar", H, E, C, device=0, mlp=mlp)
    params = torch.zeros(m.n_floats, dtype=torch.float32, device="cuda")
    grads = torch.full_like(params, float("nan"))
    for name, _ in shapes:
        m.views(params)[name].copy_(torch.from_numpy(P[name]).float())
    m.bind(params, grads)
    inputs = torch.from_numpy(X).float().cuda()
    dX = torch.full_like(inputs, float("nan"))
    m.fwd_bwd(m.build_script(graphs), inputs, dX)
    loss = m.latest_loss()
    lo, Go, dXo = M.forward_backward("bilstmchar", P, X, graphs, H)
    assert abs(loss - lo) <= TOL * abs(lo), (loss, lo)
    gv = m.views(grads.cpu())
    for name, _ in shapes:
        assert rel(gv[name].numpy(), Go[name]) <= TOL, name
    assert rel(dX.cpu().numpy(), dXo) <= TOL, "dX"


def test_bilstmchar_small():
    """M9 (reading R-38) on the GPU: character BiLSTM (H_c = E/2 = 32) on the chain recurrence feeding the word
    tagger's rare positions; ragged sentences, spellings of 2-12 characters, repeated rare words."""
    g = synth.char_tagger_batch(np.random.default_rng(600), 4, (1, 10), 64, 9, 64, rare_from=8)
    assert any(len(nd[3]) for s_ in g for nd in s_)
    _char_check(32, 64, g, 64, 601, mlp=16)


def test_bilstmchar_edge_cases():
    """No rare word (the tagger alone), a one-character spelling, a sentence of one rare word."""
    plain = [[(() if t == 0 else (t - 1,), 3 + t, t % 9, ()) for t in range(5)]]
    _char_check(32, 64, plain, 64, 602, mlp=16)
    odd = [[((), 60, 1, (7,)), ((0,), 2, 3, ()), ((1,), 61, 0, (1, 2))], [((), 62, 4, (9, 9, 9))]]
    _char_check(64, 64, odd, 64, 603, mlp=32)


def test_bilstmchar_paper_size():
    """BiLSTMwChar at Fig. 12's sizes (hidden = embedding = 256, MLP 256, character embedding 64), 16
    WikiNER-length sentences (config 'bilstmchar')."""
    g = synth.config_batch("bilstmchar", 0)
    _char_check(256, 256, g, 4096, 604, mlp=256)
