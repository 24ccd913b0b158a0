"""Pins for the traversal and layout oracles (oracle/traverse.py, oracle/layout.py,
oracle/c ora_traverse).

  * hand-derived traces on tiny graphs (tests/golden/traversal_cases.json,
    derivations written before running code) — reading R of Algorithm 1
    (PAPER.md:239-306);
  * invariants: every node has exactly one first appearance; consecutive
    path entries are adjacent in G_u unless the step was a stack pop
    (revisit) or a jump ("consecutive node appearances ...
    connected in the original graph" except at virtual edges);
  * the Python and C oracles agree on random graphs;
  * layout: edge multiset preserved exactly (north_star), CSR/CSC are
    transposes, maps are inverse bijections, WL colour multisets equal at
    every iteration, work items and partitions cover the
    edges exactly once.
"""
import json
import os
from collections import Counter

import numpy as np
import pytest

from oracle import coracle
from oracle import layout as ol
from oracle import traverse as ot
from synth import from_edge_list, random_multigraph

CASES = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "traversal_cases.json")))["cases"]


def case_graph(c):
    if "edges" in c:
        src = [a for a, b in c["edges"]] + [b for a, b in c["edges"]]
        dst = [b for a, b in c["edges"]] + [a for a, b in c["edges"]]
    else:
        src = [a for a, b in c["directed_edges"]]
        dst = [b for a, b in c["directed_edges"]]
    return from_edge_list(c["n"], src, dst)


@pytest.mark.parametrize("case", CASES, ids=[c["name"] for c in CASES])
def test_hand_traces_python(case):
    ip, ix = case_graph(case)
    r = ot.traverse(case["n"], ip, ix, window=case["window"])
    assert r["perm"].tolist() == case["perm"]
    assert r["P"].tolist() == case["P"]
    assert r["jumps"] == case["jumps"]


@pytest.mark.parametrize("case", CASES, ids=[c["name"] for c in CASES])
def test_hand_traces_c(case):
    ip, ix = case_graph(case)
    r = coracle.traverse(case["n"], ip, ix, window=case["window"])
    assert r["perm"].tolist() == case["perm"]
    assert r["P"].tolist() == case["P"]
    assert r["jumps"] == case["jumps"]


def _check_path_invariants(n, ip, ix, r):
    perm = r["perm"]
    assert sorted(perm.tolist()) == list(range(n))
    adj = ot.traversal_graph(n, ip, ix)
    P = r["P"].tolist()
    seen = set()
    nonadj = 0
    for k, v in enumerate(P):
        if k > 0 and v not in adj[P[k - 1]]:
            nonadj += 1
            # a non-adjacent step is a revisit (stack pop) or a jump to a new node
        seen.add(v)
    assert len(seen) == n
    assert len(P) - n >= 0
    # every non-adjacent step is either a revisit or a jump
    revisits = len(P) - n
    assert nonadj <= revisits + r["jumps"]


@pytest.mark.parametrize("seed", range(6))
def test_python_and_c_agree(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(5, 120))
    ip, ix = random_multigraph(seed, n, int(rng.integers(n, 6 * n)), undirected=bool(seed % 2), isolated=seed % 3)
    for window in (0, 1, 3):
        for cap in (0, 2):
            p = ot.traverse(n, ip, ix, window=window, cap=cap)
            c = coracle.traverse(n, ip, ix, window=window, cap=cap)
            assert p["perm"].tolist() == c["perm"].tolist()
            assert p["P"].tolist() == c["P"].tolist()
            assert p["jumps"] == c["jumps"]
            _check_path_invariants(n, ip, ix, p)


def wl_colour_multisets(n, ip, ix, iters=3):
    """1-WL refinement on the directed multigraph (in- and out-neighbour
    multisets); returns the multiset of colours per iteration."""
    src = np.asarray(ix, np.int64)
    dst = np.repeat(np.arange(n), np.diff(ip))
    col = [0] * n
    hist = []
    for _ in range(iters):
        ins = [[] for _ in range(n)]
        outs = [[] for _ in range(n)]
        for s, d in zip(src.tolist(), dst.tolist()):
            ins[d].append(col[s]); outs[s].append(col[d])
        sig = [(col[v], tuple(sorted(ins[v])), tuple(sorted(outs[v]))) for v in range(n)]
        table = {s: k for k, s in enumerate(sorted(set(sig)))}
        col = [table[s] for s in sig]
        hist.append(Counter(sig))
    return hist


@pytest.mark.parametrize("seed", range(4))
@pytest.mark.parametrize("k", [1, 3])
def test_layout_invariants(seed, k):
    n = 80
    ip, ix = random_multigraph(100 + seed, n, 500, undirected=bool(seed % 2), isolated=4)
    r = ot.traverse(n, ip, ix)
    L = ol.build(ip, ix, r["perm"], num_parts=k, seg_edges=8)
    perm = L["perm"]
    m = int(ip[-1])
    # multiset: (old dst, old src) pairs identical
    new_dst = np.repeat(np.arange(n), np.diff(L["indptr"]))
    got = sorted(zip(perm[new_dst].tolist(), perm[L["src"]].tolist()))
    exp = sorted(zip(np.repeat(np.arange(n), np.diff(ip)).tolist(), np.asarray(ix).tolist()))
    assert got == exp
    # eid is a bijection onto the input positions and points at the same edge
    assert sorted(L["eid"].tolist()) == list(range(m))
    assert np.array_equal(np.asarray(ix)[L["eid"]], perm[L["src"]])
    # rows sorted by (src, eid)
    for rr in range(n):
        a, b = L["indptr"][rr], L["indptr"][rr + 1]
        keys = list(zip(L["src"][a:b].tolist(), L["eid"][a:b].tolist()))
        assert keys == sorted(keys)
    # WL colour multisets equal at every iteration (relabelling is an isomorphism)
    ip2 = L["indptr"]
    assert wl_colour_multisets(n, ip, ix) == wl_colour_multisets(n, ip2, L["src"])
    # partitions: contiguous, cover all rows; edges balanced by the ceil rule
    b = L["bounds"]
    assert b[0] == 0 and b[-1] == n and np.all(np.diff(b) >= 0)
    for p in range(1, k):
        t = -(-p * m // k)
        assert L["indptr"][b[p]] >= t and (b[p] == 0 or L["indptr"][b[p] - 1] < t)
    for part in L["parts"]:
        rows = part["row_end"] - part["row_begin"]
        e = len(part["src"])
        # CSC is the transpose: cpos/csr2csc inverse, sources non-decreasing, dst valid
        assert np.array_equal(part["csr2csc"][part["cpos"]], np.arange(e))
        assert np.all(np.diff(part["src"][part["cpos"]]) >= 0)
        lip = part["indptr"]
        dl = np.repeat(np.arange(rows), np.diff(lip))
        assert np.array_equal(part["cdst"], dl[part["cpos"]])
        # items cover each CSR edge exactly once, segments <= S
        for it, nrows, ptr in ((part["fwd_items"], rows, lip), (part["bwd_items"], n, part["cindptr"])):
            cover = np.zeros(int(ptr[-1]), np.int64)
            for r_, a_, b_, s_ in it.tolist():
                assert b_ - a_ <= L["seg_edges"]
                assert ptr[r_] <= a_ <= b_ <= ptr[r_ + 1]
                cover[a_:b_] += 1
            assert np.all(cover == 1)
            assert sorted(set(it[:, 0].tolist())) == list(range(nrows))
