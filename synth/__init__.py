"""Seeded synthetic input generators shared by the oracle tests, the GPU tests and bench.py.

This module holds NO arithmetic of the method (no cell equations, no partitioning, no
scheduling): it only draws graph shapes, token ids, labels and initial parameter values
with NumPy's PCG64, so that the oracle (oracle/) and the CUDA path
(paper_conf_micro_khorasanieas18_b200/) can be fed identical inputs while sharing no code.

Graph representation (mirrors the C ABI's vpps_graph, include/vpps.h):
    a graph is a list of nodes in topological (children-first) order; node = (children, token, label)
    children : tuple of earlier node indices (tree children, or the previous LSTM step)
    token    : row of the caller's input table, or -1
    label    : class / tag / next-token id of a loss head attached to this node, or -1

Recipes (reading R-24):
  * SST-shaped binary trees: n_leaves ~ U{lo..hi}; the split point of a span of n leaves is
    ~ U{1..n-1}, recursively; leaves carry tokens ~ U{0..V_in-1}; the root carries a label
    ~ U{0..C-1} (root-only head, reading R-3).  (parse trees of SST.)
  * Variable-length sentences (LSTM chains): length ~ U{lo..hi}; token_t ~ U{0..V-1};
    LM target label_t = token_{t+1}, last position unlabelled.  (BASELINE.json config 1/3.)
  * Tagger sentences: length ~ U{lo..hi}; labels ~ U{0..T-1} at every position.
  * Parameters: Glorot-uniform matrices, biases U(-0.1, 0.1); input table U(-0.1, 0.1) (R-21).
"""
from __future__ import annotations

import numpy as np

__all__ = [
    "rng_for", "sst_tree", "tree_batch", "chain", "chain_batch", "tagger_batch",
    "init_params", "input_table", "config_batch", "CONFIGS",
]


def rng_for(config_id: int, batch_idx: int) -> np.random.Generator:
    """Config k, batch b -> PCG64 seeded with SeedSequence([1000+k, b])."""
    return np.random.Generator(np.random.PCG64(np.random.SeedSequence([1000 + config_id, batch_idx])))


def sst_tree(rng: np.random.Generator, n_leaves: int, vocab: int, n_classes: int):
    """One binary tree with n_leaves leaves, children-first order, label at the root only."""
    nodes: list[tuple[tuple[int, ...], int, int]] = []

    def build(n: int) -> int:
        if n == 1:
            nodes.append(((), int(rng.integers(0, vocab)), -1))
            return len(nodes) - 1
        k = int(rng.integers(1, n))          # split point in {1..n-1}
        left = build(k)
        right = build(n - k)
        nodes.append(((left, right), -1, -1))
        return len(nodes) - 1

    root = build(n_leaves)
    ch, tok, _ = nodes[root]
    nodes[root] = (ch, tok, int(rng.integers(0, n_classes)))
    return nodes


def tree_batch(rng, batch: int, leaves=(5, 50), vocab=4096, n_classes=5):
    return [sst_tree(rng, int(rng.integers(leaves[0], leaves[1] + 1)), vocab, n_classes)
            for _ in range(batch)]


def chain(rng: np.random.Generator, length: int, vocab: int, lm: bool = True, n_tags: int = 0):
    """An LSTM chain: node t has the single child t-1; LM labels are next tokens."""
    toks = rng.integers(0, vocab, size=length)
    if lm:
        labels = [int(toks[t + 1]) for t in range(length - 1)] + [-1]
    else:
        labels = [int(x) for x in rng.integers(0, n_tags, size=length)]
    return [((t - 1,) if t > 0 else (), int(toks[t]), labels[t]) for t in range(length)]


def chain_batch(rng, batch: int, lengths=(5, 60), vocab=1000):
    return [chain(rng, int(rng.integers(lengths[0], lengths[1] + 1)), vocab, lm=True)
            for _ in range(batch)]


def tagger_batch(rng, batch: int, lengths=(5, 60), vocab=4096, n_tags=9):
    return [chain(rng, int(rng.integers(lengths[0], lengths[1] + 1)), vocab, lm=False, n_tags=n_tags)
            for _ in range(batch)]


def td_pyramid(rng: np.random.Generator, length: int, vocab: int, n_classes: int):
    """A TD-RNN graph over a sentence of `length` tokens (reading R-36): level 0 the tokens,
    node i of level k composes nodes i and i+1 of level k-1 (each inner node of a level below the top has
    two parents), the single top node carries the sentence label.  Nodes are listed level by level."""
    toks = rng.integers(0, vocab, size=length)
    nodes = [((), int(t), -1) for t in toks]
    prev = list(range(length))
    for _ in range(1, length):
        cur = []
        for i in range(len(prev) - 1):
            nodes.append(((prev[i], prev[i + 1]), -1, -1))
            cur.append(len(nodes) - 1)
        prev = cur
    top = prev[0]
    nodes[top] = (nodes[top][0], nodes[top][1], int(rng.integers(0, n_classes)))
    return nodes


def td_batch(rng, batch: int, lengths=(5, 30), vocab=4096, n_classes=5):
    return [td_pyramid(rng, int(rng.integers(lengths[0], lengths[1] + 1)), vocab, n_classes) for _ in range(batch)]


def init_params(shapes, rng: np.random.Generator, dtype=np.float64):
    """shapes: ordered list of (name, shape). Glorot-uniform for 2-D, U(-0.1, 0.1) for 1-D."""
    out = {}
    for name, shape in shapes:
        if len(shape) == 2:
            lim = np.sqrt(6.0 / (shape[0] + shape[1]))
            out[name] = rng.uniform(-lim, lim, size=shape).astype(dtype)
        else:
            out[name] = rng.uniform(-0.1, 0.1, size=shape).astype(dtype)
    return out


def input_table(rng: np.random.Generator, n_rows: int, dim: int, dtype=np.float64):
    return rng.uniform(-0.1, 0.1, size=(n_rows, dim)).astype(dtype)


def spelling(word: int, n_chars: int = 64, lengths=(2, 12)):
    """Deterministic synthetic spelling of a word id (BiLSTMwChar): a length in `lengths` and
    character ids in [0, n_chars), drawn from a generator seeded by the word id alone, so every occurrence
    of a word is spelled the same way."""
    r = np.random.default_rng(np.random.SeedSequence([0x5EED, int(word)]))
    n = int(r.integers(lengths[0], lengths[1] + 1))
    return tuple(int(c) for c in r.integers(0, n_chars, size=n))


def char_tagger_batch(rng, batch: int, lengths=(5, 60), vocab=4096, n_tags=9, n_chars=64, rare_from=None):
    """BiLSTMwChar sentences (reading R-38): tagger chains whose word ids follow a Zipf-like law (WikiNER-
    style frequencies); ids >= rare_from (default: the top quarter of the vocabulary, the words seen fewer
    than 5 times in a corpus of this law) are rare and carry their spelling as a fourth node field."""
    rare_from = (3 * vocab) // 4 if rare_from is None else rare_from
    out = []
    for _ in range(batch):
        n = int(rng.integers(lengths[0], lengths[1] + 1))
        toks = np.minimum((rng.pareto(1.0, size=n) * vocab / 64).astype(np.int64), vocab - 1)
        labs = rng.integers(0, n_tags, size=n)
        out.append([((t - 1,) if t > 0 else (), int(toks[t]), int(labs[t]),
                     spelling(int(toks[t]), n_chars) if toks[t] >= rare_from else ())
                    for t in range(n)])
    return out


# BASELINE.json configs (SURVEY §8 "Configs"); 'tgt' is the north_star target.
CONFIGS = {
    "c1": dict(cell="lstm", H=32, E=32, C=16, V=16, batch=4, lengths=(2, 5)),
    "c2": dict(cell="childsum", H=128, E=128, C=5, V=4096, batch=16, leaves=(5, 50)),
    "c3": dict(cell="lstm", H=256, E=256, C=1000, V=1000, batch=16, lengths=(5, 60)),
    "c4": dict(cell="bilstm", H=512, E=512, C=9, V=4096, batch=16, lengths=(5, 60), mlp=256),
    "c5": dict(cell="binary", H=1024, E=1024, C=5, V=4096, batch=64, leaves=(5, 50)),
    "tgt": dict(cell="binary", H=256, E=256, C=5, V=4096, batch=16, leaves=(5, 50)),
    # paper's other workloads (Fig. 12: hidden = embedding = 512), SST-length sentences
    "tdrnn": dict(cell="tdrnn", H=512, E=512, C=5, V=4096, batch=16, lengths=(5, 30)),
    # BiLSTMwChar (Fig. 12: hidden = embedding = 256, MLP 256, character embedding 64), WikiNER-length sentences
    "bilstmchar": dict(cell="bilstmchar", H=256, E=256, C=9, V=4096, batch=16, lengths=(5, 60), mlp=256,
                       Ec=64, Vc=64),
}
_CONFIG_IDS = {"c1": 1, "c2": 2, "c3": 3, "c4": 4, "c5": 5, "tgt": 6, "tdrnn": 7, "bilstmchar": 8}


def config_batch(name: str, batch_idx: int, batch: int | None = None, **over):
    """Graphs of batch `batch_idx` for a named config (optionally overriding the batch size)."""
    cfg = dict(CONFIGS[name])
    cfg.update(over)
    b = cfg["batch"] if batch is None else batch
    rng = rng_for(_CONFIG_IDS[name], batch_idx)
    if cfg["cell"] in ("binary", "childsum"):
        return tree_batch(rng, b, cfg["leaves"], cfg["V"], cfg["C"])
    if cfg["cell"] == "bilstmchar":
        return char_tagger_batch(rng, b, cfg["lengths"], cfg["V"], cfg["C"], cfg["Vc"])
    if cfg["cell"] == "tdrnn":
        return td_batch(rng, b, cfg["lengths"], cfg["V"], cfg["C"])
    if cfg["cell"] == "lstm":
        return [chain(rng, int(rng.integers(cfg["lengths"][0], cfg["lengths"][1] + 1)), cfg["V"], lm=True)
                for _ in range(b)]
    return tagger_batch(rng, b, cfg["lengths"], cfg["V"], cfg["C"])
