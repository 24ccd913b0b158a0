"""Tiny seeded graphs for tests (numpy only; no method arithmetic).

Multigraphs with the structures the method must handle: duplicate edges,
self-loops, isolated and zero-in-degree nodes, directed edges, several
components.  CSR rows are destinations; within a row edges keep input order.
"""
from __future__ import annotations

import numpy as np


def from_edge_list(n: int, src, dst):
    """(src[e] -> dst[e]) pairs -> CSR by destination, stable in input order."""
    src = np.asarray(src, dtype=np.int64)
    dst = np.asarray(dst, dtype=np.int64)
    order = np.argsort(dst, kind="stable")
    indptr = np.zeros(n + 1, dtype=np.int64)
    np.add.at(indptr, dst + 1, 1)
    indptr = np.cumsum(indptr).astype(np.int64)
    return indptr, src[order].astype(np.int32)


def to_edge_list(indptr, indices):
    deg = np.diff(indptr)
    dst = np.repeat(np.arange(len(indptr) - 1), deg)
    return np.asarray(indices, dtype=np.int64), dst


def random_multigraph(seed: int, n: int, m: int, undirected: bool = False, p_self: float = 0.05,
                      p_dup: float = 0.1, isolated: int = 0):
    """Random multigraph on n nodes with about m directed edges."""
    rng = np.random.default_rng(seed)
    hi = max(1, n - isolated)
    pairs = []
    target = m // 2 if undirected else m
    while len(pairs) < target:
        r = rng.random()
        if pairs and r < p_dup:
            pairs.append(pairs[rng.integers(len(pairs))])
        elif r < p_dup + p_self:
            v = int(rng.integers(hi))
            pairs.append((v, v))
        else:
            pairs.append((int(rng.integers(hi)), int(rng.integers(hi))))
    src, dst = [], []
    for a, b in pairs:
        src.append(a); dst.append(b)
        if undirected:
            src.append(b); dst.append(a)
    return from_edge_list(n, src, dst)
