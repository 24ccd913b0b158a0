"""Faithful path-band representation (traversal variant F of
§8(c)-c1b) and GAT attention over it, fp64.  Test infrastructure only (see
oracle/__init__.py).

The paper's own representation (Fig. 7): one
traversal builds a path P of node *appearances* (with revisits); the graph is
then stored as a band of width omega along P — an edge is represented by the
pair of appearances (t - o, t), 1 <= o <= omega, that covers it — so the
neighbour rows of appearance t are the 2 omega appearances around it, read as
a sequential stream instead of a gather.

Traversal F differs from R (oracle/traverse.py) in four
places, followed here in that order:
  (1) coverage: every G_u edge starts uncovered; N(v) = the neighbours of v
      over uncovered edges (Table IV's "unvisited neighbors").
      When any node x is appended to P (every tier), each uncovered edge
      {x, u} with u among the previous omega entries of P becomes covered
      (its owner is the pair (t, o), u = P[t - o]) and leaves both N sets;
  (2) tier-1 candidates: the first K entries of N(curr) in id order — they
      may be visited nodes (a revisit along a real edge);
  (3) score(v) = |adj(v) ∩ {last omega entries of P}| (Eq. (2) literally,
      revisits in the window); ties -> smallest id;
  (4) termination: U = ∅ and covered / |E_u| >= theta (
      theta = 1 here: every edge covered).
Tiers 2 and 3 and the start rule are R's (R15, R17): tier 2 pops
stack entries whose N is empty, then pops the top (a revisit; every
appearance whose N is non-empty after its coverage step is pushed); tier 3
jumps to the unvisited node minimising (deg_u is even, id).  Reading R-band-1
(DESIGN.md): once U = ∅ with edges still uncovered and both tiers 1 and 2
empty, tier 3 takes the node with a non-empty N by the same key (c1b is silent;
the paper's loop condition, continues until the ratio is met).

Band layout of the directed input multiset (exact, north_star): a covered G_u
edge {x, u} with owner (t, o) carries the multiplicities of x <- u and u <- x
in the input; self-loops x -> x (not in G_u) are attached to the first
appearance of x.  GAT over the band: appearance t aggregates the in-edges of
P[t] that its band pairs own — sources P[t - o] through pairs (t, o) and
P[t + o] through pairs (t + o, o), plus its self-loops — into a partial softmax
state (max, sum, weighted row sum); the partial states of a node's
appearances are merged (online-softmax combine).  The result is graph
attention over the same multiset, so it equals oracle/gat.py exactly (up to
summation order): that equality, the coverage invariant and the revisit bound
pin this file (tests/test_oracle_band.py).
"""
from __future__ import annotations

import numpy as np

from .traverse import auto_window, traversal_graph


def traverse_faithful(n, indptr, indices, window=0, cap=0):
    """-> dict(P, owner, omega, K, jumps, virtual).  owner[t] = offsets o (ascending) of the
    G_u edges {P[t], P[t - o]} covered when P[t] was appended."""
    m = int(np.asarray(indptr)[-1]) if n else 0
    omega = window if window > 0 else auto_window(n, m)
    K = cap if cap > 0 else 32
    adj = traversal_graph(n, indptr, indices)
    adjset = [set(a) for a in adj]
    N = [set(a) for a in adj]                  # uncovered neighbours
    n_edges = sum(len(a) for a in adj) // 2
    covered = 0
    visited = [False] * n
    P, owner, stk = [], [], []
    tier3_picks = 0

    def append(x):
        nonlocal covered
        t = len(P)
        own = []
        for o in range(1, omega + 1):
            if t - o < 0:
                break
            u = P[t - o]
            if u != x and u in N[x]:           # (1) coverage by the later endpoint
                N[x].discard(u)
                N[u].discard(x)
                covered += 1
                own.append(o)
        P.append(x)
        owner.append(own)
        visited[x] = True

    def score(v):                              # (3)
        win = P[-omega:]
        return sum(1 for w in win if w in adjset[v])

    def tier3():
        pool = [v for v in range(n) if not visited[v]]
        if not pool:                           # R-band-1
            pool = [v for v in range(n) if N[v]]
        best = None
        for v in pool:
            key = (len(adj[v]) % 2 == 0, v)
            if best is None or key < best[0]:
                best = (key, v)
        return best[1]

    if n == 0:
        return {"P": np.zeros(0, np.int32), "owner": [], "omega": omega, "K": K, "jumps": 0, "virtual": 0}
    curr = tier3(); tier3_picks += 1
    append(curr)
    if N[curr]:
        stk.append(curr)
    virtual = 0
    while not (all(visited) and covered >= n_edges):   # (4), theta = 1
        C = sorted(N[curr])[:K]                          # (2)
        if C:
            best = C[0]
            bs = score(best)
            for v in C[1:]:
                sv = score(v)
                if sv > bs:
                    best, bs = v, sv
            curr = best
        else:
            while stk and not N[stk[-1]]:
                stk.pop()
            if stk:
                nxt = stk.pop()                          # tier 2: revisit
            else:
                nxt = tier3(); tier3_picks += 1          # tier 3: jump
            if nxt not in adjset[curr]:
                virtual += 1
            curr = nxt
        append(curr)
        if N[curr]:
            stk.append(curr)
    return {"P": np.asarray(P, np.int32), "owner": owner, "omega": omega, "K": K,
            "jumps": tier3_picks - 1, "virtual": virtual}


def band_layout(n, indptr, indices, trav):
    """Directed multiplicities on the band pairs.  -> dict(P, pairs, self_loops) with
    pairs = list of (t, o, c_fwd, c_bwd): c_fwd = #edges P[t-o] -> P[t] (destination P[t]),
    c_bwd = #edges P[t] -> P[t-o]; self_loops[v] = #edges v -> v."""
    indptr = np.asarray(indptr)
    cnt = {}
    self_loops = np.zeros(n, np.int64)
    for i in range(n):
        for e in range(int(indptr[i]), int(indptr[i + 1])):
            j = int(indices[e])
            if j == i:
                self_loops[i] += 1
            else:
                cnt[(i, j)] = cnt.get((i, j), 0) + 1      # destination i, source j
    P = trav["P"]
    pairs = []
    for t, offs in enumerate(trav["owner"]):
        x = int(P[t])
        for o in offs:
            u = int(P[t - o])
            pairs.append((t, o, cnt.get((x, u), 0), cnt.get((u, x), 0)))
    return {"P": P, "pairs": pairs, "self_loops": self_loops}


def band_gat_forward(n, band, Wh, a_l, a_r, slope=0.2):
    """GAT forward over the band (H heads): per appearance partial softmax states over the
    in-edges its pairs own, merged per node.  Wh [n, H, F], a_l / a_r [H, F] float64.
    -> dict(out [n, H, F], lse [n, H])."""
    Wh = np.asarray(Wh, np.float64)
    H, F = Wh.shape[1], Wh.shape[2]
    s = np.float64(np.float32(slope))
    el = np.einsum("nhf,hf->nh", Wh, a_l)
    er = np.einsum("nhf,hf->nh", Wh, a_r)
    P = band["P"]
    L = len(P)
    # the in-edges of each appearance: (source node, multiplicity)
    inlist = [[] for _ in range(L)]
    for t, o, c_fwd, c_bwd in band["pairs"]:
        if c_fwd:
            inlist[t].append((int(P[t - o]), c_fwd))      # P[t-o] -> P[t]
        if c_bwd:
            inlist[t - o].append((int(P[t]), c_bwd))      # P[t] -> P[t-o]
    first = {}
    for t in range(L):
        first.setdefault(int(P[t]), t)
    for v, t in first.items():
        if band["self_loops"][v]:
            inlist[t].append((v, int(band["self_loops"][v])))
    # partial states per appearance (step 1), merged per node in appearance order (step 2)
    parts = [[] for _ in range(n)]
    for t in range(L):
        x = int(P[t])
        if not inlist[t]:
            continue
        z = np.array([[el[x, h] + er[j, h] for h in range(H)] for j, _ in inlist[t]])
        sc = np.where(z > 0, z, s * z)
        c = np.array([m for _, m in inlist[t]], np.float64)
        mx = sc.max(axis=0)
        w = c[:, None] * np.exp(sc - mx)
        lsum = w.sum(axis=0)
        acc = np.einsum("eh,ehf->hf", w, np.stack([Wh[j] for j, _ in inlist[t]]))
        parts[x].append((mx, lsum, acc))
    out = np.zeros((n, H, F))
    lse = np.full((n, H), -np.inf)
    for x in range(n):
        if not parts[x]:
            continue
        M = np.max([p[0] for p in parts[x]], axis=0)
        Ls = sum(p[1] * np.exp(p[0] - M) for p in parts[x])
        A = sum(p[2] * np.exp(p[0] - M)[:, None] for p in parts[x])
        out[x] = A / Ls[:, None]
        lse[x] = M + np.log(Ls)
    return {"out": out, "lse": lse}
