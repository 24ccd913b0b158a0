"""The paper's own workload: block-diagonal batches of
small graphs shaped like Table II, with and without the 20%
edge dropping of PAPER.md:413.

CPU (`not gpu`): the generator matches Table II and is simple/symmetric/
block-diagonal; edge dropping removes exactly round(0.2 * pairs) pairs per
graph; the oracle on a batch equals the oracle on each graph alone (a GAT layer
never mixes components, PAPER.md:51 aggregates over N(i) only); the product
reorganiser is bit-exact vs the oracle reorganiser on a batch.
GPU (`gpu`): libmega.so vs the oracle, element by element, on batches at the
paper's hidden sizes 64 and 128."""
import numpy as np
import pytest

import synth
from oracle import coracle
from synth.batch import SHAPES, drop_edges, make_batch
from synth.tiny import to_edge_list
from paper_conf_icdcs_dengr24_b200 import mega as M
from tests.test_layout_product import _compare, _oracle_layout


def _pairs(ip, ix):
    src, dst = to_edge_list(ip, ix)
    return src, dst


@pytest.mark.parametrize("name", sorted(SHAPES))
def test_batch_matches_table_ii(name):
    ip, ix, gptr = make_batch(name, 256, seed=7)
    n_mean, m_mean, _ = SHAPES[name]
    G = len(gptr) - 1
    assert G == 256 and gptr[-1] == len(ip) - 1 and ip[-1] == len(ix)
    assert abs((len(ip) - 1) / G - n_mean) <= 0.1 * n_mean
    assert abs(len(ix) / G - m_mean) <= 0.1 * m_mean
    src, dst = _pairs(ip, ix)
    assert np.all(src != dst)                                       # no self-loops
    key = src * (len(ip) - 1) + dst
    assert len(np.unique(key)) == len(key)                          # simple
    assert np.array_equal(np.sort(key), np.sort(dst * (len(ip) - 1) + src))   # symmetric
    gs = np.searchsorted(gptr, src, side="right")
    assert np.array_equal(gs, np.searchsorted(gptr, dst, side="right"))       # block-diagonal
    if name == "csl":
        assert np.all(np.diff(ip) == 4) and np.all(np.diff(gptr) == 41)


def test_batch_is_seeded():
    a = make_batch("zinc", 64, seed=3)
    b = make_batch("zinc", 64, seed=3)
    c = make_batch("zinc", 64, seed=4)
    assert all(np.array_equal(x, y) for x, y in zip(a, b))
    assert not np.array_equal(a[1], c[1]) or not np.array_equal(a[0], c[0])


@pytest.mark.parametrize("name", ["aqsol", "zinc", "csl"])
def test_edge_dropping(name):
    ip, ix, gptr = make_batch(name, 64, seed=11)
    ip2, ix2 = drop_edges(ip, ix, gptr, 0.2, seed=12)
    n = len(ip) - 1
    s1, d1 = _pairs(ip, ix)
    s2, d2 = _pairs(ip2, ix2)
    k1, k2 = set(zip(s1.tolist(), d1.tolist())), set(zip(s2.tolist(), d2.tolist()))
    assert k2 <= k1 and len(k2) == len(ix2)
    assert all((d, s) in k2 for s, d in k2)                          # still symmetric
    for g in range(len(gptr) - 1):
        lo, hi = gptr[g], gptr[g + 1]
        p1 = sum(1 for s, d in k1 if lo <= d < hi and s < d)
        p2 = sum(1 for s, d in k2 if lo <= d < hi and s < d)
        assert p1 - p2 == int(round(0.2 * p1))
    assert len(ip2) == n + 1


def _inputs(seed, n, H, F):
    rng = np.random.default_rng(seed)
    Wh = rng.standard_normal((n, H, F))
    a_l = rng.standard_normal((H, F)) / np.sqrt(F)
    a_r = rng.standard_normal((H, F)) / np.sqrt(F)
    g = rng.standard_normal((n, H, F))
    return Wh, a_l, a_r, g


@pytest.mark.parametrize("name", ["zinc", "cycles"])
def test_oracle_batch_equals_per_graph(name):
    """Block independence: the batch oracle restricted to graph b equals the oracle
    run on graph b alone (forward out/lse and backward grad_feat); the parameter
    gradients are the sums of the per-graph ones."""
    ip, ix, gptr = make_batch(name, 12, seed=5)
    n, H, F = len(ip) - 1, 4, 8
    Wh, a_l, a_r, g = _inputs(9, n, H, F)
    fb = coracle.gat_forward(ip, ix, Wh, a_l, a_r)
    bb = coracle.gat_backward(ip, ix, Wh, a_l, a_r, g, fwd=fb)
    gal = np.zeros((H, F))
    gar = np.zeros((H, F))
    for b in range(len(gptr) - 1):
        lo, hi = int(gptr[b]), int(gptr[b + 1])
        sip = ip[lo:hi + 1] - ip[lo]
        six = ix[ip[lo]:ip[hi]] - lo
        f = coracle.gat_forward(sip, six, Wh[lo:hi], a_l, a_r)
        bw = coracle.gat_backward(sip, six, Wh[lo:hi], a_l, a_r, g[lo:hi], fwd=f)
        np.testing.assert_allclose(fb["out"][lo:hi], f["out"], rtol=1e-12, atol=1e-12)
        np.testing.assert_array_equal(np.isfinite(fb["lse"][lo:hi]), np.isfinite(f["lse"]))
        np.testing.assert_allclose(bb["grad_feat"][lo:hi], bw["grad_feat"], rtol=1e-12, atol=1e-12)
        gal += bw["grad_attn_l"].reshape(H, F)
        gar += bw["grad_attn_r"].reshape(H, F)
    np.testing.assert_allclose(bb["grad_attn_l"].reshape(H, F), gal, rtol=1e-10, atol=1e-12)
    np.testing.assert_allclose(bb["grad_attn_r"].reshape(H, F), gar, rtol=1e-10, atol=1e-12)


@pytest.mark.parametrize("cfg_name", ["zinc-b64", "aqsol-b128-drop20", "csl-b128"])
def test_layout_bit_exact_on_batches(cfg_name):
    cfg = synth.get_config(cfg_name)
    ip, ix, _ = synth.make_graph(cfg)
    assert (len(ip) - 1, len(ix)) == (cfg.n, cfg.m)
    lay = M.mega_preprocess(ip, ix, num_parts=2)
    ref, r = _oracle_layout(ip, ix, "traversal", 0, 0, 2, 0)
    _compare(lay, ref, r)


@pytest.mark.gpu
@pytest.mark.parametrize("dtype", ["fp32", "bf16"])
@pytest.mark.parametrize("cfg_name,H,F", [("zinc-b64", 8, 16), ("zinc-b128", 8, 8), ("aqsol-b128-drop20", 8, 16),
                                          ("csl-b128", 8, 16), ("cycles-b128", 4, 32)])
def test_gpu_parity_batches(cuda_device, dtype, cfg_name, H, F):
    from tests import gpu_harness as hz
    cfg = synth.get_config(cfg_name)
    ip, ix, _ = synth.make_graph(cfg)
    Wh, a_l, a_r, g = hz.inputs(cfg.seed, cfg.n, H, F, dtype == "bf16")
    lay = M.mega_preprocess(ip, ix, seg_edges=8)
    got = hz.run_attention(lay, Wh, a_l, a_r, g, dtype)
    f = coracle.gat_forward(ip, ix, Wh, a_l, a_r)
    ref = {**f, **coracle.gat_backward(ip, ix, Wh, a_l, a_r, g, fwd=f)}
    hz.check(got, ref, dtype, graph=(ip, ix, Wh, a_l, a_r, g))
