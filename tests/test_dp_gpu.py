"""Data parallelism through the real CUDA path (north_star): two ranks on cuda:0 with
the gloo backend (CUDA tensors), each running libvpps on its shard of one global batch —
vpps_fwd_bwd (dataflow path: leaf GEMM, vpps_df, gradient GEMM) -> all_reduce(sum) of the flat gradient ->
vpps_sgd_step — against the FP64 oracle on the union batch (the summed loss makes shards additive, L205).
"""
import os
import socket

import numpy as np
import pytest

import synth
from oracle import models as M

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
H = E = 256
C, V = 5, 4096
LR, WD = 0.05, 1e-3


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _setup(seed=5):
    rng = np.random.default_rng(seed)
    from paper_conf_micro_khorasanieas18_b200 import vpps
    shapes = vpps.param_shapes("binary", H, E, C)
    P = synth.init_params(shapes, rng)
    X = synth.input_table(rng, V, E)
    graphs = synth.config_batch("tgt", 30)
    return shapes, P, X, graphs


def _worker(rank, world, port, out):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_micro_khorasanieas18_b200 import dp, vpps
    shapes, P, X, graphs = _setup()
    m = vpps.Model("binary", H, E, C, device=0, cluster=16, dataflow=True)
    params = torch.zeros(m.n_floats, dtype=torch.float32, device="cuda:0")
    grads = torch.zeros_like(params)
    for name, _ in shapes:
        m.views(params)[name].copy_(torch.from_numpy(P[name]).float())
    m.bind(params, grads)
    inputs = torch.from_numpy(X).float().cuda()
    mine = dp.shard(graphs, rank, world)
    s = m.build_script(mine)
    m.fwd_bwd(s, inputs)
    local = grads.clone()
    dist.all_reduce(grads, op=dist.ReduceOp.SUM)      # gloo on CUDA tensors (NCCL in the bench)
    m.sgd_step(LR, WD)
    torch.cuda.synchronize()
    loss = dp.global_loss(m.latest_loss(), "cpu")
    out[rank] = (local.double().cpu().numpy(), grads.double().cpu().numpy(), params.cpu().numpy().copy(), loss,
                 len(mine))
    dist.destroy_process_group()


def test_dp_two_ranks_real_kernels():
    import torch.multiprocessing as mp
    world = 2
    out = mp.Manager().dict()
    mp.spawn(_worker, args=(world, _free_port(), out), nprocs=world, join=True)
    from paper_conf_micro_khorasanieas18_b200 import vpps
    shapes, P, X, graphs = _setup()
    lo, Go, _ = M.forward_backward("binary", P, X.astype(np.float32).astype(np.float64), graphs, H)
    Pn = M.sgd(P, Go, LR, WD)
    m = vpps.Model("binary", H, E, C, plan_only=True)
    assert out[0][4] + out[1][4] == len(graphs) and min(out[0][4], out[1][4]) > 0
    # shard gradients sum to the union's, and the reduced gradient equals the oracle's
    g_sum = out[0][0] + out[1][0]
    for r in range(world):
        assert np.array_equal(out[r][1], out[0][1])
        gv = m.views(out[r][1])
        for name, _ in shapes:
            ref = Go[name]
            assert np.abs(gv[name] - ref).max() <= 1e-4 * np.abs(ref).max(), name
    assert np.abs(g_sum - out[0][1]).max() <= 1e-6 * np.abs(out[0][1]).max()
    # replicas identical after the step, and equal to the oracle's SGD step (1e-4 of the step + FP32 rounding)
    assert np.array_equal(out[0][2], out[1][2])
    pv = m.views(out[0][2].astype(np.float64))
    for name, _ in shapes:
        step = Pn[name] - P[name]
        bound = 1e-4 * np.abs(step).max() + 2.0 ** -22 * np.abs(Pn[name]).max()
        assert np.abs(pv[name] - Pn[name]).max() <= bound, name
    assert abs(out[0][3] - lo) <= 1e-4 * abs(lo) and out[0][3] == out[1][3]
