"""Writes tests/golden/full_<case>.npz: the FP64 oracle's loss and sampled gradient entries for the
BASELINE.json configurations at their full sizes, where the oracle needs minutes (SURVEY §8(d) configs
3, 4, 5).  Calls only oracle/ and synth/ (no product code): the summed loss is additive over the graphs of
a batch, so the batch is split over worker processes and their results summed.

    python tools/make_golden.py [case ...]        (cases: c5, c4, c3; default all)

Stored per case: the input recipe (config, batch index, seed), the loss, and per gradient tensor (and dX)
its max |value| (the R-22 denominator) with 2048 sampled entries (flat index, value) — 1984 uniformly
drawn plus the 64 largest in magnitude (dX: drawn from its nonzero rows)."""
import multiprocessing as mp
import os
import sys

os.environ.setdefault("OPENBLAS_NUM_THREADS", "1")
os.environ.setdefault("OMP_NUM_THREADS", "1")
os.environ.setdefault("MKL_NUM_THREADS", "1")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import synth  # noqa: E402
from oracle import models as M  # noqa: E402

# case -> (cell, H, E, C, V, mlp, config name, batch index, batch override, seed of params / input table)
CASES = {
    "c5": ("binary", 1024, 1024, 5, 4096, 256, "c5", 0, None, 63),
    "c4": ("bilstm", 512, 512, 9, 4096, 256, "c4", 1, None, 73),
    "c3": ("lstm", 256, 256, 1000, 1000, 256, "c3", 3, 64, 84),
}
N_SAMPLE, N_TOP = 2048, 64


def inputs(case):
    cell, H, E, C, V, mlp, cfg, b, batch, seed = CASES[case]
    graphs = synth.config_batch(cfg, b, batch=batch)
    rng = np.random.default_rng(seed)
    P = synth.init_params(M.param_shapes(cell, H, E, C, mlp), rng)
    X = synth.input_table(rng, V, E)
    # the device computes with FP32 parameters and inputs: the oracle takes the same values
    P = {k: v.astype(np.float32).astype(np.float64) for k, v in P.items()}
    X = X.astype(np.float32).astype(np.float64)
    return graphs, P, X


def _part(args):
    case, lo, hi = args
    graphs, P, X = inputs(case)
    cell, H = CASES[case][0], CASES[case][1]
    return M.forward_backward(cell, P, X, graphs[lo:hi], H)


def sample(rng, flat, nonzero_only=False):
    pool = np.flatnonzero(flat) if nonzero_only else np.arange(flat.size)
    top = np.argsort(-np.abs(flat))[:N_TOP]
    rand = rng.choice(pool, size=min(N_SAMPLE - N_TOP, pool.size), replace=False)
    idx = np.unique(np.concatenate([top, rand]))
    return idx.astype(np.int64), flat[idx]


def make(case, procs):
    graphs, P, X = inputs(case)
    n = len(graphs)
    cuts = np.linspace(0, n, min(procs, n) + 1).astype(int)
    with mp.Pool(len(cuts) - 1) as pool:
        parts = pool.map(_part, [(case, int(a), int(b)) for a, b in zip(cuts[:-1], cuts[1:])])
    loss = sum(p[0] for p in parts)
    G = {k: sum(p[1][k] for p in parts) for k in parts[0][1]}
    dX = sum(p[2] for p in parts)
    rng = np.random.default_rng(12345)
    out = dict(loss=np.float64(loss))
    for k in sorted(G):
        flat = G[k].ravel()
        idx, val = sample(rng, flat)
        out[f"{k}__idx"], out[f"{k}__val"], out[f"{k}__max"] = idx, val, np.abs(flat).max()
    idx, val = sample(rng, dX.ravel(), nonzero_only=True)
    out["dX__idx"], out["dX__val"], out["dX__max"] = idx, val, np.abs(dX).max()
    path = os.path.join(ROOT, "tests", "golden", f"full_{case}.npz")
    np.savez_compressed(path, **out)
    print(case, "loss", loss, "->", path)


if __name__ == "__main__":
    cases = sys.argv[1:] or list(CASES)
    for c in cases:
        make(c, os.cpu_count() or 1)
