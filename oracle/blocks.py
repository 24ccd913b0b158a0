"""L2 blocking of the node order — plain definition.  Integer only.

Test infrastructure only (see oracle/__init__.py).

Not from the paper: this is our B200 addition to the reorganiser (DESIGN.md
R24).  MEGA's traversal makes neighbours adjacent in the path (PAPER.md:188,
310), which helps a cache of a few rows; the B200's 126 MB L2 holds ~10^5
feature rows, so the order should also keep each *L2-sized* run of
destinations on a source set that fits there.  The blocks come from
size-constrained label propagation on G_u (the traversal graph of
oracle/traverse.py), then the traversal order is stably regrouped by block:

  * visit order: ascending (deg_u(v), v);
  * label(v) = v initially, size(l) = |{v : label(v) = l}|;
  * a sweep visits every v with deg_u(v) > 0 once, in visit order, and sets
    label(v) to the argmax over l in {label(v)} ∪ {label(u) : u ∈ adj(v),
    size(l) < B} of (cnt(l), l == label(v), -l), where
    cnt(l) = |{u ∈ adj(v) : label(u) = l}|; sizes update immediately;
  * sweeps stop after `sweeps` (0 = 10) or once a sweep changes fewer than
    n/1000 labels (changed * 1000 < n);
  * blocks are ranked by the first position any member holds in the base
    order; the new order lists the blocks in rank order, each block's nodes
    in base order.
"""
from __future__ import annotations

from collections import Counter

import numpy as np

from .traverse import traversal_graph


def propagate(n, indptr, indices, B, sweeps=0):
    """-> (label list, sweeps run).  Follows the module docstring literally."""
    adj = traversal_graph(n, indptr, indices)
    T = sweeps if sweeps > 0 else 10
    label = list(range(n))
    size = Counter(label)
    visit = sorted(range(n), key=lambda v: (len(adj[v]), v))
    run = 0
    for _ in range(T):
        run += 1
        changed = 0
        for v in visit:
            if not adj[v]:
                continue
            cnt = Counter(label[u] for u in adj[v])
            cur = label[v]
            cands = [cur] + [l for l in cnt if l != cur and size[l] < B]
            best = max(cands, key=lambda l: (cnt.get(l, 0), l == cur, -l))
            if best != cur:
                size[cur] -= 1
                size[best] += 1
                label[v] = best
                changed += 1
        if changed * 1000 < n:
            break
    return label, run


def regroup(base_perm, label):
    """Stable regroup of the base order by block, blocks in first-position order."""
    first = {}
    for r, v in enumerate(base_perm):
        first.setdefault(label[v], r)
    order = sorted(range(len(base_perm)), key=lambda r: (first[label[base_perm[r]]], r))
    return np.asarray([base_perm[r] for r in order], np.int32), len(first)


def blocked_order(n, indptr, indices, base_perm, B, sweeps=0):
    """-> dict(perm, label, num_blocks, sweeps)."""
    label, run = propagate(n, indptr, indices, B, sweeps)
    perm, nb = regroup([int(v) for v in base_perm], label)
    return {"perm": perm, "label": np.asarray(label, np.int64), "num_blocks": nb, "sweeps": run}
