"""Host-side product tests (no GPU): libmega.so loads, exports every symbol
include/mega.h declares, validates its inputs, and mega_preprocess (a1) is
bit-exact against the independent oracle reorganiser (oracle/traverse.py,
oracle/c ora_traverse, oracle/layout.py)."""
import os
import re

import numpy as np
import pytest

import synth
from oracle import coracle
from oracle import blocks as ob
from oracle import layout as ol
from oracle import traverse as ot
from paper_conf_icdcs_dengr24_b200 import mega as M

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "mega.h")).read()
    declared = set(re.findall(r"^\s*(?:[\w\s\*]+?)\b(mega_\w+)\s*\(", hdr, flags=re.M))
    assert len(declared) >= 17
    L = M.lib()
    for name in sorted(declared):
        assert hasattr(L, name), name
    assert M.mega_abi_version() == 2


def test_invalid_inputs_are_rejected():
    with pytest.raises(M.MegaError) as e:
        M.mega_preprocess(np.array([0, 2, 1]), np.array([0, 1], np.int32))
    assert e.value.status == 2  # INVALID_GRAPH (not monotone)
    with pytest.raises(M.MegaError) as e:
        M.mega_preprocess(np.array([0, 1]), np.array([5], np.int32))
    assert e.value.status == 2  # index out of range
    with pytest.raises(M.MegaError) as e:
        M.mega_preprocess(np.array([0, 1]), np.array([0], np.int32), candidate_cap=100)
    assert e.value.status == 1


def _oracle_layout(ip, ix, order, window, cap, parts, seg, seed=0, block_rows=0):
    n = len(ip) - 1
    if order == "traversal":
        r = ot.traverse(n, ip, ix, window=window, cap=cap) if n <= 3000 else coracle.traverse(n, ip, ix, window, cap)
        perm = r["perm"]
    elif order == "identity":
        perm, r = ot.order_identity(n), None
    elif order == "degree":
        perm, r = ot.order_degree(n, ip), None
    else:
        perm, r = ot.order_random(n, seed), None
    if block_rows > 0:
        if n <= 3000:
            perm = ob.blocked_order(n, ip, ix, perm, block_rows)["perm"]
        else:
            label, _ = coracle.l2_blocks(ip, ix, block_rows)
            perm, _ = ob.regroup([int(v) for v in perm], label.tolist())
    return ol.build(ip, ix, perm, num_parts=parts, seg_edges=seg), r


def _compare(layout, ref, r):
    st = layout.stats()
    assert st["seg_edges"] == ref["seg_edges"]
    if r is not None:
        assert st["path_length"] == len(r["P"]) if "P" in r else st["path_length"] == r["path_length"]
        assert st["jumps"] == r["jumps"]
    for p, part in enumerate(ref["parts"]):
        v = layout.view(p)
        assert np.array_equal(v["perm"], ref["perm"])
        assert np.array_equal(v["new_of_old"], ref["new_of_old"])
        assert np.array_equal(v["bounds"], ref["bounds"])
        assert (v["row_begin"], v["row_end"]) == (part["row_begin"], part["row_end"])
        for k in ("indptr", "src", "eid", "cindptr", "cdst", "cpos", "csr2csc", "fwd_items", "fwd_splits",
                  "bwd_items", "bwd_splits"):
            assert np.array_equal(v[k], part[k]), k


@pytest.mark.parametrize("seed", range(5))
@pytest.mark.parametrize("order", ["traversal", "identity", "degree", "random"])
def test_bit_exact_vs_oracle_tiny(seed, order):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(3, 150))
    ip, ix = synth.random_multigraph(seed, n, int(rng.integers(1, 8 * n)), undirected=bool(seed % 2),
                                     isolated=seed % 4)
    window, cap, parts, seg = [(0, 0, 1, 0), (2, 3, 2, 4), (1, 1, 3, 7), (5, 0, 4, 2), (0, 64, 1, 1)][seed]
    lay = M.mega_preprocess(ip, ix, window=window, candidate_cap=cap, order=order, seg_edges=seg, num_parts=parts,
                            seed=1234 + seed)
    ref, r = _oracle_layout(ip, ix, order, window, cap, parts, seg, seed=1234 + seed)
    _compare(lay, ref, r if order == "traversal" else None)


@pytest.mark.parametrize("name", ["cora", "pubmed"])
def test_bit_exact_vs_oracle_configs(name):
    cfg = synth.CONFIGS[name]
    ip, ix, _ = synth.make_graph(cfg)
    lay = M.mega_preprocess(ip, ix, num_parts=2)
    ref, r = _oracle_layout(ip, ix, "traversal", 0, 0, 2, 0)
    _compare(lay, ref, r)
    st = lay.stats()
    assert st["tile_unique_sources"] == ol.tile_unique_sources(ref["indptr"], ref["src"])
    assert st["window"] == ot.auto_window(cfg.n, cfg.m)


@pytest.mark.slow
def test_bit_exact_vs_oracle_arxiv():
    cfg = synth.CONFIGS["arxiv"]
    ip, ix, _ = synth.make_graph(cfg)
    lay = M.mega_preprocess(ip, ix, num_parts=4, seg_edges=64)
    ref, r = _oracle_layout(ip, ix, "traversal", 0, 0, 4, 64)
    _compare(lay, ref, r)


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("order", ["traversal", "degree", "random"])
def test_bit_exact_blocked_vs_oracle_tiny(seed, order):
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(3, 200))
    ip, ix = synth.random_multigraph(100 + seed, n, int(rng.integers(1, 8 * n)), undirected=bool(seed % 2),
                                     isolated=seed % 3)
    B = [1, 2, 5, 17, 64, 1000][seed]
    lay = M.mega_preprocess(ip, ix, order=order, num_parts=1 + seed % 3, seg_edges=1 + seed, block_rows=B,
                            seed=7 + seed)
    ref, r = _oracle_layout(ip, ix, order, 0, 0, 1 + seed % 3, 1 + seed, seed=7 + seed, block_rows=B)
    _compare(lay, ref, r if order == "traversal" else None)
    st = lay.stats()
    label, sweeps = coracle.l2_blocks(ip, ix, B)
    assert st["block_sweeps"] == sweeps and st["num_blocks"] == len(set(label.tolist()))


@pytest.mark.parametrize("name", ["cora", "pubmed"])
def test_bit_exact_blocked_vs_oracle_configs(name):
    cfg = synth.CONFIGS[name]
    ip, ix, _ = synth.make_graph(cfg)
    B = M.auto_block_rows(cfg.dim * 2, 2 * 1024 * 1024)  # a small L2 so that the configs split into blocks
    lay = M.mega_preprocess(ip, ix, num_parts=2, block_rows=B)
    ref, r = _oracle_layout(ip, ix, "traversal", 0, 0, 2, 0, block_rows=B)
    _compare(lay, ref, r)
    assert lay.stats()["num_blocks"] > 1


def test_l2_blocking_improves_block_scale_reuse():
    """On a products-shaped graph the blocked order should need far fewer
    distinct sources per L2-sized run of destinations than the plain traversal."""
    cfg = synth.scaled(synth.CONFIGS["products"], 40000, 600000)
    ip, ix, _ = synth.make_graph(cfg)
    B = 4000

    def distinct_per_run(lay):
        v = lay.view(0)
        tot = 0
        for r0 in range(0, cfg.n, B):
            a, b = int(v["indptr"][r0]), int(v["indptr"][min(cfg.n, r0 + B)])
            tot += np.unique(v["src"][a:b]).size
        return tot
    plain = distinct_per_run(M.mega_preprocess(ip, ix))
    blocked = distinct_per_run(M.mega_preprocess(ip, ix, block_rows=B))
    assert blocked < 0.7 * plain, (blocked, plain)


def test_save_load_roundtrip(tmp_path):
    ip, ix = synth.random_multigraph(3, 60, 300, undirected=True)
    lay = M.mega_preprocess(ip, ix, num_parts=2, seg_edges=5)
    p = str(tmp_path / "l.mega")
    M.mega_layout_save(lay, p)
    lay2 = M.mega_layout_load(p)
    assert lay.stats() == lay2.stats()
    for part in range(2):
        a, b = lay.view(part), lay2.view(part)
        for k in a:
            assert np.array_equal(np.asarray(a[k]), np.asarray(b[k])), k
    raw = bytearray(open(p, "rb").read())
    raw[100] ^= 0xFF
    open(p, "wb").write(bytes(raw))
    with pytest.raises(M.MegaError) as e:
        M.mega_layout_load(p)
    assert e.value.status == 7


def test_mega_ordering_improves_locality():
    """The traversal's order should give more source reuse per 64-row tile than
    the random input order (the premise of PAPER.md:188, 310)."""
    cfg = synth.scaled(synth.CONFIGS["products"], 40000, 600000)
    ip, ix, _ = synth.make_graph(cfg)
    mega_ = M.mega_preprocess(ip, ix).stats()
    ident = M.mega_preprocess(ip, ix, order="identity").stats()
    assert mega_["tile_unique_sources"] < 0.9 * ident["tile_unique_sources"]
