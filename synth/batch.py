"""mega-synth v1, batch recipe: the paper's own workload.

Test/bench input generator with none of the method's arithmetic.  The paper
evaluates on mini-batches of many small graphs (Table II;
batch sizes 64/128/256, hidden 64/128: PAPER.md:156, 346, 369), which DGL
batches as one block-diagonal graph.  We draw seeded graphs shaped like each
dataset's Table II row (mean nodes, mean directed edges; sparsity = m/n^2):

  zinc    23 nodes,  50 edges  molecule: random backbone tree + ring closures
  aqsol   18 nodes,  36 edges  molecule
  csl     41 nodes, 164 edges  cycle C_41 with one skip-link length (4-regular)
  cycles  49 nodes,  88 edges  one 6-cycle, a tree hung off it, isolated rest

All graphs are undirected (both directions emitted), simple (no self-loops,
no duplicate pairs).  `drop_edges` is the paper's edge dropping
("20% of edges are randomly dropped within every graph"),
read as dropping round(frac * pairs) undirected pairs per graph, both
directions (DESIGN.md R-drop).
"""
from __future__ import annotations

import numpy as np

from synth.tiny import from_edge_list

# Table II: mean nodes, mean directed edges, generator kind
SHAPES = {
    "zinc": (23, 50, "molecule"),
    "aqsol": (18, 36, "molecule"),
    "csl": (41, 164, "csl"),
    "cycles": (49, 88, "cycles"),
}
CSL_SKIPS = (2, 3, 4, 5, 6, 9, 11, 12, 13, 16)


def _pairs(rng, kind, n_mean, m_mean):
    """-> (n, list of undirected pairs (u, v), u != v, no repeats)."""
    if kind == "csl":
        n = 41
        s = int(rng.choice(CSL_SKIPS))
        return n, [(i, (i + 1) % n) for i in range(n)] + [(i, (i + s) % n) for i in range(n)]
    lo, hi = max(3, round(0.6 * n_mean)), round(1.4 * n_mean)
    n = int(rng.integers(lo, hi + 1))
    target = max(1, round(n * m_mean / (2.0 * n_mean)))
    seen, out = set(), []

    def add(u, v):
        k = (min(u, v), max(u, v))
        if u != v and k not in seen:
            seen.add(k)
            out.append((u, v))

    if kind == "molecule":
        for v in range(1, n):                     # chain-like backbone tree
            add(int(rng.integers(max(0, v - 3), v)), v)
        tries = 0
        while len(out) < target and tries < 50 * n:   # ring closures
            tries += 1
            u = int(rng.integers(0, n))
            add(u, (u + int(rng.integers(4, 7))) % n)
    else:                                         # cycles
        for i in range(6):
            add(i, (i + 1) % 6)
        for v in range(6, n):
            if len(out) >= target:
                break                             # the rest stay isolated (in-degree 0)
            add(int(rng.integers(0, v)), v)
    return n, out


def make_batch(name: str, num_graphs: int, seed: int):
    """Block-diagonal batch of `num_graphs` graphs shaped like Table II's `name` row.
    -> (indptr int64[n+1], indices int32[m], graph_ptr int64[num_graphs+1])."""
    n_mean, m_mean, kind = SHAPES[name]
    rng = np.random.default_rng(seed)
    src, dst, gptr = [], [], [0]
    for _ in range(num_graphs):
        n, pairs = _pairs(rng, kind, n_mean, m_mean)
        off = gptr[-1]
        for u, v in pairs:
            src += [off + u, off + v]
            dst += [off + v, off + u]
        gptr.append(off + n)
    ip, ix = from_edge_list(gptr[-1], np.array(src, np.int64), np.array(dst, np.int64))
    return ip, ix, np.array(gptr, np.int64)


def drop_edges(indptr, indices, graph_ptr, frac: float, seed: int):
    """Drop round(frac * pairs_g) undirected pairs of every graph g (both directions),
    chosen uniformly without replacement.  Input must be symmetric and simple."""
    rng = np.random.default_rng(seed)
    deg = np.diff(indptr)
    dst = np.repeat(np.arange(len(indptr) - 1, dtype=np.int64), deg)
    src = np.asarray(indices, np.int64)
    upper = src < dst                               # one entry per undirected pair
    gid = np.searchsorted(graph_ptr, dst, side="right") - 1
    drop = set()
    for g in range(len(graph_ptr) - 1):
        idx = np.nonzero(upper & (gid == g))[0]
        k = int(round(frac * len(idx)))
        for e in rng.choice(idx, size=k, replace=False) if k else ():
            drop.add((int(src[e]), int(dst[e])))
    keep = np.array([(min(s, d), max(s, d)) not in drop for s, d in zip(src.tolist(), dst.tolist())], bool)
    return from_edge_list(len(indptr) - 1, src[keep], dst[keep])
