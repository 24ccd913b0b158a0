"""Traversal R — the deterministic reading of MEGA's Algorithm 1. fp-free, integer.

Test infrastructure only (see oracle/__init__.py).

Follows PAPER.md §III-B "Graph Reorganization" in the paper's order and
notation: one traversal of the graph that picks, at each step,
the candidate maximising its correlation with the last omega path entries,
Eq. (1)/(2), from three candidate tiers
(PAPER.md:231-233), with a stack of visited nodes that still have unvisited
neighbours (Alg. 1) and jumps when
both pools are empty.  Readings of garbled/ambiguous
points are DESIGN.md R8-R19:

  * the traversal graph G_u is the symmetrised simple view (i != j, deduped),
    adjacency in ascending id order ("minor adjustments");
  * CORRELATE(v) = |adj(v) ∩ W| where W = the last omega FIRST appearances
    (PAPER.md:244 garbled; Eq. (2));
  * tier 1 = the first K unvisited neighbours of curr in id order
    (PAPER.md:231 line 1); argmax ties -> smallest id;
  * tier 2 = pop stale stack entries, then pop the top (a revisit,
    PAPER.md:280 garbled);
  * tier 3 / start = the unvisited node minimising (deg is even, id)
    ("minimize ... commencing a new path from nodes with an even
    degree"; CORRELATE over U is identically 0 there);
  * omega = clamp(round(m/n), 1, 64), K = 32;
  * loop until every node has a first appearance (U = ∅).

This oracle scans adjacency lists naively from the start (no compaction); it
is meant for small graphs.  oracle/c/oracle.c holds the same loop in C.
"""
from __future__ import annotations

from collections import deque

import numpy as np


def auto_window(n: int, m: int) -> int:
    """omega = clamp(round(m/n), 1, 64), round half up (R16)."""
    if n <= 0:
        return 1
    return int(min(64, max(1, (2 * m + n) // (2 * n))))


def traversal_graph(n, indptr, indices):
    """G_u: {i, j} for every edge j -> i with i != j, deduplicated, sorted."""
    adj = [set() for _ in range(n)]
    indptr = np.asarray(indptr)
    for i in range(n):
        for e in range(int(indptr[i]), int(indptr[i + 1])):
            j = int(indices[e])
            if j != i:
                adj[i].add(j)
                adj[j].add(i)
    return [sorted(a) for a in adj]


def traverse(n, indptr, indices, window=0, cap=0):
    """-> dict(perm, P, jumps, window, cap).  perm[r] = old id of new id r."""
    m = int(np.asarray(indptr)[-1]) if n else 0
    omega = window if window > 0 else auto_window(n, m)
    K = cap if cap > 0 else 32
    adj = traversal_graph(n, indptr, indices)
    visited = [False] * n
    score = [0] * n            # |adj(v) ∩ W| for unvisited v
    W = deque()                # last omega first appearances
    perm, P, stk = [], [], []
    tier3_picks = 0

    def has_unvisited(v):
        return any(not visited[u] for u in adj[v])

    def visit(v):
        visited[v] = True
        perm.append(v)
        for u in adj[v]:
            if not visited[u]:
                score[u] += 1
        W.append(v)
        if len(W) > omega:
            o = W.popleft()
            for u in adj[o]:
                if not visited[u]:
                    score[u] -= 1

    def tier3():
        best = None
        for v in range(n):                         # min (deg is even, id)
            if not visited[v]:
                key = (len(adj[v]) % 2 == 0, v)
                if best is None or key < best[0]:
                    best = (key, v)
        return best[1]

    if n == 0:
        return {"perm": np.zeros(0, np.int32), "P": np.zeros(0, np.int32), "jumps": 0,
                "window": omega, "cap": K}
    curr = tier3(); tier3_picks += 1
    visit(curr)
    P.append(curr)
    if has_unvisited(curr):
        stk.append(curr)
    while len(perm) < n:
        C = [u for u in adj[curr] if not visited[u]][:K]          # tier 1
        if C:
            best = C[0]
            for v in C[1:]:
                if score[v] > score[best]:
                    best = v
            curr = best
            visit(curr)
        else:
            while stk and not has_unvisited(stk[-1]):
                stk.pop()
            if stk:
                curr = stk.pop()                                   # tier 2: revisit
            else:
                curr = tier3(); tier3_picks += 1                   # tier 3: jump
                visit(curr)
        P.append(curr)
        if has_unvisited(curr):
            stk.append(curr)
    return {"perm": np.asarray(perm, np.int32), "P": np.asarray(P, np.int32),
            "jumps": tier3_picks - 1, "window": omega, "cap": K}


def order_identity(n):
    return np.arange(n, dtype=np.int32)


def order_degree(n, indptr):
    """Ablation: stable sort by (-in-degree, id)."""
    deg = np.diff(np.asarray(indptr, np.int64))
    return np.lexsort((np.arange(n), -deg)).astype(np.int32)


def order_random(n, seed):
    """Ablation: Fisher-Yates driven by splitmix64(seed) draws (i-th output)."""
    perm = list(range(n))
    MASK = (1 << 64) - 1

    def mix(z):
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK
        return z ^ (z >> 31)

    for i in range(n - 1, 0, -1):
        u = mix((seed + (n - 1 - i + 1) * 0x9E3779B97F4A7C15) & MASK)
        j = (u >> 11) % (i + 1)
        perm[i], perm[j] = perm[j], perm[i]
    return np.asarray(perm, np.int32)
