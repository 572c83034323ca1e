"""world_size-2 gloo test (CPU) of the data-parallel step ordering in paper_conf_micro_khorasanieas18_b200.dp.

The CUDA fwd_bwd / sgd kernels cannot run here, so a stand-in model computes its shard's gradient with the
oracle and applies the update with the same formula; what is under test is the sharding, the all-reduce
and the ordering: Σ_r grads(shard_r) == grads(union), and every rank ends with bitwise-identical params.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth
from oracle import models as M

H, E, C, V = 4, 4, 3, 12


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class OracleModel:
    """Stand-in with the vpps.Model call surface used by dp_step."""

    def __init__(self, P, X, grads, params):
        self.P, self.X, self.grads, self.params = P, X, grads, params
        self.names = [n for n, _ in M.param_shapes("binary", H, E, C)]

    def fwd_bwd(self, graphs, inputs, d_inputs, stream=None):
        _, G, _ = M.forward_backward("binary", self.P, self.X, graphs, H)
        self.grads.copy_(torch.from_numpy(np.concatenate([G[n].ravel() for n in self.names])))

    def sgd_step(self, lr, wd, stream=None):
        self.params -= lr * (self.grads + wd * self.params)


def _worker(rank, world, port, out):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_micro_khorasanieas18_b200 import dp
    rng = np.random.default_rng(0)
    P = synth.init_params(M.param_shapes("binary", H, E, C), rng)
    X = synth.input_table(rng, V, E)
    graphs = synth.tree_batch(np.random.default_rng(1), 5, (1, 6), V, C)
    names = [n for n, _ in M.param_shapes("binary", H, E, C)]
    params = torch.from_numpy(np.concatenate([P[n].ravel() for n in names])).clone()
    grads = torch.zeros_like(params)
    m = OracleModel(P, X, grads, params)
    mine = dp.shard(graphs, rank, world)
    dp.dp_step(m, mine, None, None, grads, lr=0.1, weight_decay=0.01)
    loss_local = M.forward_backward("binary", P, X, mine, H)[0]
    out[rank] = (grads.numpy().copy(), params.numpy().copy(), dp.global_loss(loss_local, "cpu"))
    dist.destroy_process_group()


def test_dp_two_ranks_gloo():
    world = 2
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(world, _free_port(), out), nprocs=world, join=True)
    rng = np.random.default_rng(0)
    P = synth.init_params(M.param_shapes("binary", H, E, C), rng)
    X = synth.input_table(rng, V, E)
    graphs = synth.tree_batch(np.random.default_rng(1), 5, (1, 6), V, C)
    loss, G, _ = M.forward_backward("binary", P, X, graphs, H)
    names = [n for n, _ in M.param_shapes("binary", H, E, C)]
    g_union = np.concatenate([G[n].ravel() for n in names])
    p_new = np.concatenate([M.sgd(P, G, 0.1, 0.01)[n].ravel() for n in names])
    for r in range(world):
        np.testing.assert_allclose(out[r][0], g_union, rtol=0, atol=1e-12)
        np.testing.assert_allclose(out[r][1], p_new, rtol=0, atol=1e-12)
        assert abs(out[r][2] - loss) < 1e-10
    assert np.array_equal(out[0][1], out[1][1])        # replicas identical after the step


def test_shard_covers_batch_once():
    from paper_conf_micro_khorasanieas18_b200 import dp
    items = list(range(17))
    for world in (1, 2, 3, 8):
        got = [x for r in range(world) for x in dp.shard(items, r, world)]
        assert got == items
