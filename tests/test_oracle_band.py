"""Pins for the faithful path-band oracle (oracle/band.py, traversal
variant F of §8(c)-c1b).

  * the star trace of SURVEY Appendix C item 1 (hand-derived there before any
    code): centre 0, leaves 1-4, omega = 1 -> P = [1,0,2,0,3,0,4], 2 revisits —
    below PAPER.md:219's sum ceil(d/omega) - n = 3 (reported, never asserted);
  * theta = 1: every G_u edge is covered exactly once, by a pair (t, o) whose
    appearances are its two endpoints; every node appears;
  * the valid revisit bound |P| - n >= max(sum ceil(d_i / 2 omega), ceil(|E_u| / omega)) - n
    (an appearance has <= 2 omega band neighbours; each edge is covered by its later
    endpoint against <= omega predecessors);
  * the band stores the directed multiset exactly (multiplicities + self-loops);
  * GAT over the band equals graph attention (oracle/gat.py, itself pinned by
    dense masked attention) on random multigraphs with duplicates, self-loops,
    isolated nodes, directed edges — the band is a re-representation, not an
    approximation.
"""
from collections import Counter

import numpy as np
import pytest

from oracle import band as ob
from oracle import gat as og
from oracle import traverse as ot
from synth import from_edge_list, random_multigraph


def undirected(n, edges):
    src = [a for a, b in edges] + [b for a, b in edges]
    dst = [b for a, b in edges] + [a for a, b in edges]
    return from_edge_list(n, src, dst)


def test_star_trace():
    ip, ix = undirected(5, [(0, 1), (0, 2), (0, 3), (0, 4)])
    tr = ob.traverse_faithful(5, ip, ix, window=1)
    assert tr["P"].tolist() == [1, 0, 2, 0, 3, 0, 4]
    assert len(tr["P"]) - 5 == 2
    assert tr["owner"] == [[], [1], [1], [], [1], [], [1]]


def test_path_is_one_pass():
    ip, ix = undirected(4, [(0, 1), (1, 2), (2, 3)])
    tr = ob.traverse_faithful(4, ip, ix, window=2)
    assert tr["P"].tolist() == [0, 1, 2, 3] and tr["virtual"] == 0


@pytest.mark.parametrize("seed", range(12))
@pytest.mark.parametrize("omega", [1, 2, 4])
def test_coverage_and_bound(seed, omega):
    ip, ix = random_multigraph(seed, 30, 90, undirected=seed % 2 == 0, isolated=2)
    n = len(ip) - 1
    tr = ob.traverse_faithful(n, ip, ix, window=omega)
    P = tr["P"]
    adj = ot.traversal_graph(n, ip, ix)
    Eu = {(min(i, j), max(i, j)) for i in range(n) for j in adj[i]}
    owned = Counter()
    for t, offs in enumerate(tr["owner"]):
        for o in offs:
            assert 1 <= o <= omega and t - o >= 0
            a, b = int(P[t]), int(P[t - o])
            owned[(min(a, b), max(a, b))] += 1
    assert set(owned) == Eu and all(c == 1 for c in owned.values())
    assert set(P.tolist()) == set(range(n))
    deg = [len(a) for a in adj]
    lb = max(sum(-(-d // (2 * omega)) for d in deg), -(-len(Eu) // omega))
    assert len(P) >= lb


@pytest.mark.parametrize("seed", range(6))
def test_band_preserves_multiset(seed):
    ip, ix = random_multigraph(100 + seed, 40, 160, undirected=seed % 2 == 1, isolated=3)
    n = len(ip) - 1
    band = ob.band_layout(n, ip, ix, ob.traverse_faithful(n, ip, ix, window=3))
    P = band["P"]
    got = Counter()
    for t, o, cf, cb in band["pairs"]:
        x, u = int(P[t]), int(P[t - o])
        got[(x, u)] += cf        # (destination, source)
        got[(u, x)] += cb
    for v in range(n):
        got[(v, v)] += int(band["self_loops"][v])
    want = Counter((i, int(ix[e])) for i in range(n) for e in range(int(ip[i]), int(ip[i + 1])))
    assert +got == want


@pytest.mark.parametrize("seed,H,F", [(0, 1, 4), (1, 2, 3), (2, 4, 2), (3, 2, 5)])
def test_band_gat_equals_graph_attention(seed, H, F):
    ip, ix = random_multigraph(200 + seed, 35, 140, undirected=seed % 2 == 0, isolated=2)
    n = len(ip) - 1
    rng = np.random.default_rng(seed)
    Wh = rng.standard_normal((n, H, F))
    a_l, a_r = rng.standard_normal((H, F)), rng.standard_normal((H, F))
    band = ob.band_layout(n, ip, ix, ob.traverse_faithful(n, ip, ix, window=2))
    got = ob.band_gat_forward(n, band, Wh, a_l, a_r)
    ref = og.gat_forward(ip, ix, Wh, a_l, a_r)
    np.testing.assert_allclose(got["out"], ref["out"], rtol=1e-12, atol=1e-12)
    fin = np.isfinite(ref["lse"])
    assert np.array_equal(fin, np.isfinite(got["lse"]))
    np.testing.assert_allclose(got["lse"][fin], ref["lse"][fin], rtol=1e-12, atol=1e-12)
