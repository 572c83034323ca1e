"""Data parallelism for the VPPS step (BASELINE.json north_star).

The paper is single-GPU.  Graphs of a batch are independent and the loss is their sum
(L205), so the step shards naturally: rank r runs its own persistent kernel on its contiguous slice of
the global batch with a full weight replica, the flat gradient buffers are summed with one NCCL
all-reduce over NVLink, and every rank applies the same SGD update (L129, L197).  The all-reduce is the
only collective on the data path.  The per-rank math never leaves libvpps; this module only orders the
three calls and does the sharding arithmetic.
"""
from __future__ import annotations


def shard(graphs, rank: int, world: int):
    """Contiguous slice of the global batch for `rank` (sizes differ by at most one graph)."""
    n = len(graphs)
    lo = (n * rank) // world
    hi = (n * (rank + 1)) // world
    return graphs[lo:hi]


def dp_step(model, script, inputs, d_inputs, grads, lr: float, weight_decay: float, group=None, stream=None):
    """vpps_fwd_bwd -> all_reduce(sum) of the flat gradient -> vpps_sgd_step on every rank."""
    import torch.distributed as dist
    model.fwd_bwd(script, inputs, d_inputs, stream=stream)
    dist.all_reduce(grads, op=dist.ReduceOp.SUM, group=group)
    model.sgd_step(lr, weight_decay, stream=stream)


def global_loss(local_loss: float, device, group=None) -> float:
    """Summed batch loss over ranks (the super-graph's aggregated loss, L205)."""
    import torch
    import torch.distributed as dist
    t = torch.tensor([local_loss], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return float(t[0])
