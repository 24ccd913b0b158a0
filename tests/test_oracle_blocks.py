"""Pins for the L2-blocking oracle (oracle/blocks.py, oracle/c ora_l2_blocks;
DESIGN.md R24): hand-derived label-propagation traces, planted partitions
whose answer is known, and invariants of the regrouped order."""
import numpy as np
import pytest

import synth
from oracle import blocks as ob
from oracle import coracle


def _undirected(n, pairs):
    src = [a for a, b in pairs] + [b for a, b in pairs]
    dst = [b for a, b in pairs] + [a for a, b in pairs]
    return synth.from_edge_list(n, src, dst)


K4 = [(0, 1), (0, 2), (0, 3), (1, 2), (1, 3), (2, 3)]


def test_k4_one_block_when_it_fits():
    # visit order 0,1,2,3 (all deg 3): 0 takes the smallest of three count-1
    # labels (1); 1 keeps its own label on the tie; 2 and 3 see label 1 twice.
    ip, ix = _undirected(4, K4)
    label, sweeps = ob.propagate(4, ip, ix, B=4)
    assert label == [1, 1, 1, 1]
    assert sweeps == 2  # sweep 1 changes 3 labels, sweep 2 none


def test_k4_size_cap_two():
    # B = 2: 0 -> 1 (block {0,1} full); 2: label 1 has count 2 but is full, so
    # 2 takes 3 (count 1 beats its own label's count 0); 3 keeps 3 (tie).
    ip, ix = _undirected(4, K4)
    label, sweeps = ob.propagate(4, ip, ix, B=2)
    assert label == [1, 1, 3, 3]
    assert sweeps == 2
    r = ob.blocked_order(4, ip, ix, [3, 2, 1, 0], B=2)
    assert r["perm"].tolist() == [3, 2, 1, 0]  # block {2,3} first (position 0), then {0,1}, base order kept
    r = ob.blocked_order(4, ip, ix, [0, 2, 1, 3], B=2)
    assert r["perm"].tolist() == [0, 1, 2, 3]
    assert r["num_blocks"] == 2


def test_b1_keeps_base_order():
    ip, ix = synth.random_multigraph(4, 40, 200, undirected=True)
    base = np.random.default_rng(0).permutation(40)
    r = ob.blocked_order(40, ip, ix, base, B=1)
    assert r["perm"].tolist() == base.tolist()
    assert r["num_blocks"] == 40


def _ring_of_cliques(c, s):
    pairs = []
    for q in range(c):
        nodes = [q * s + i for i in range(s)]
        pairs += [(a, b) for i, a in enumerate(nodes) for b in nodes[i + 1:]]
        pairs.append((q * s + s - 1, ((q + 1) % c) * s))  # one bridge to the next clique
    return pairs


@pytest.mark.parametrize("c,s", [(3, 5), (7, 6), (12, 9)])
def test_planted_cliques_recovered(c, s):
    n = c * s
    ip, ix = _undirected(n, _ring_of_cliques(c, s))
    for B in (s, s + 3, n):
        label, _ = ob.propagate(n, ip, ix, B=B)
        blocks = {}
        for v, l in enumerate(label):
            blocks.setdefault(l, set()).add(v)
        assert sorted(map(sorted, blocks.values())) == [list(range(q * s, q * s + s)) for q in range(c)]
        lc, _ = coracle.l2_blocks(ip, ix, B)
        assert lc.tolist() == label


@pytest.mark.parametrize("seed", range(6))
def test_invariants_random(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(5, 120))
    ip, ix = synth.random_multigraph(seed, n, int(rng.integers(1, 6 * n)), undirected=bool(seed % 2),
                                     isolated=seed % 3)
    base = rng.permutation(n)
    B = int(rng.integers(1, 12))
    r = ob.blocked_order(n, ip, ix, base, B=B)
    perm, label = r["perm"], r["label"]
    assert sorted(perm.tolist()) == list(range(n))
    sizes = np.bincount(label, minlength=n)
    assert sizes.max() <= B
    pos = {int(v): i for i, v in enumerate(base)}
    lab_seq = label[perm]
    # blocks are contiguous runs, ranked by first base position, base order inside
    runs = [lab_seq[0]] + [lab_seq[i] for i in range(1, n) if lab_seq[i] != lab_seq[i - 1]]
    assert len(runs) == len(set(runs)) == r["num_blocks"]
    firsts = [min(pos[int(v)] for v in perm if label[v] == l) for l in runs]
    assert firsts == sorted(firsts)
    for l in runs:
        members = [pos[int(v)] for v in perm if label[v] == l]
        assert members == sorted(members)
    lc, sw = coracle.l2_blocks(ip, ix, B)
    assert lc.tolist() == label.tolist() and sw == r["sweeps"]
