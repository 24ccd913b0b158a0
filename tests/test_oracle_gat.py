"""Pins for the GAT oracle (oracle/gat.py and oracle/c via coracle.py).

Each test checks the oracle against something other than itself:
  * the dense "global attention" formulation with non-edges masked to -inf
    (Fig. 1a: graph attention is global attention restricted
    to the real edges), via torch.softmax / logsumexp in fp64, duplicates as
    +log(multiplicity) (R5);
  * torch autograd of that dense formulation (backward);
  * central finite differences;
  * closed forms and special cases (a = 0 -> row-normalised SpMM via
    scipy.sparse; slope = 1 cancels el; in-degree 1 -> out = Wh_src);
  * invariants (softmax sums to 1, sum_in ds = 0, sum del = sum der,
    relabelling equivariance — north_star);
  * a hand-computed golden example (tests/golden/gat_tiny.json).
"""
import json
import os

import numpy as np
import pytest
import scipy.sparse as sp
import torch

from oracle import coracle
from oracle import gat as og
from synth import bf16_round, from_edge_list, random_multigraph

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _inputs(seed, n, H, F):
    rng = np.random.default_rng(seed)
    Wh = rng.standard_normal((n, H, F)).astype(np.float32)
    a_l = (rng.standard_normal((H, F)) / np.sqrt(F)).astype(np.float32)
    a_r = (rng.standard_normal((H, F)) / np.sqrt(F)).astype(np.float32)
    g = rng.standard_normal((n, H, F)).astype(np.float32)
    return Wh, a_l, a_r, g


class PyImpl:
    name = "python"
    fwd = staticmethod(og.gat_forward)
    bwd = staticmethod(og.gat_backward)


class CImpl:
    name = "c"
    fwd = staticmethod(coracle.gat_forward)
    bwd = staticmethod(coracle.gat_backward)


@pytest.fixture(params=[PyImpl, CImpl], ids=["python", "c"])
def impl(request):
    return request.param


def dense_reference(indptr, indices, Wh, a_l, a_r, g, slope=og.SLOPE):
    """Global attention on the dense n x n score matrix, non-edges at -inf."""
    n, H, F = Wh.shape
    mult = np.zeros((n, n))
    deg = np.diff(indptr)
    dst = np.repeat(np.arange(n), deg)
    np.add.at(mult, (dst, np.asarray(indices)), 1.0)
    Wh_t = torch.tensor(Wh, dtype=torch.float64, requires_grad=True)
    al_t = torch.tensor(a_l, dtype=torch.float64, requires_grad=True)
    ar_t = torch.tensor(a_r, dtype=torch.float64, requires_grad=True)
    el = torch.einsum("nhf,hf->nh", Wh_t, al_t)
    er = torch.einsum("nhf,hf->nh", Wh_t, ar_t)
    z = el.T[:, :, None] + er.T[:, None, :]                       # [H, i, j]
    s = torch.nn.functional.leaky_relu(z, negative_slope=slope)
    logm = torch.log(torch.tensor(mult, dtype=torch.float64))      # -inf on non-edges
    s = s + logm[None]
    has = torch.tensor(deg > 0)
    att = torch.softmax(torch.where(has[None, :, None], s, torch.zeros_like(s)), dim=-1)
    att = torch.where(has[None, :, None], att, torch.zeros_like(att))
    out = torch.einsum("hij,jhf->ihf", att, Wh_t)
    lse = torch.logsumexp(s, dim=-1).T                             # -inf for empty rows
    loss = (out * torch.tensor(g, dtype=torch.float64)).sum()
    loss.backward()
    return {"out": out.detach().numpy(), "lse": lse.detach().numpy(), "grad_feat": Wh_t.grad.numpy(),
            "grad_attn_l": al_t.grad.numpy(), "grad_attn_r": ar_t.grad.numpy()}


GRAPHS = [
    ("directed-multi", lambda: random_multigraph(1, 9, 30, undirected=False, isolated=2)),
    ("undirected-multi", lambda: random_multigraph(2, 12, 40, undirected=True)),
    ("selfloops-dups", lambda: from_edge_list(5, [0, 0, 1, 1, 2, 3, 3, 4], [1, 1, 1, 0, 2, 4, 4, 3])),
]


@pytest.mark.parametrize("H,F", [(1, 1), (2, 3), (4, 8)])
@pytest.mark.parametrize("gname,gfn", GRAPHS, ids=[g[0] for g in GRAPHS])
def test_matches_dense_global_attention(impl, gname, gfn, H, F):
    indptr, indices = gfn()
    n = len(indptr) - 1
    Wh, a_l, a_r, g = _inputs(7, n, H, F)
    ref = dense_reference(indptr, indices, Wh, a_l, a_r, g)
    f = impl.fwd(indptr, indices, Wh, a_l, a_r)
    b = impl.bwd(indptr, indices, Wh, a_l, a_r, g)
    np.testing.assert_allclose(f["out"], ref["out"], rtol=1e-12, atol=1e-12)
    fin = np.isfinite(ref["lse"])
    assert np.array_equal(fin, np.isfinite(f["lse"]))
    np.testing.assert_allclose(f["lse"][fin], ref["lse"][fin], rtol=1e-12, atol=1e-12)
    assert np.all(f["lse"][~fin] == -np.inf)
    for k in ("grad_feat", "grad_attn_l", "grad_attn_r"):
        np.testing.assert_allclose(b[k], ref[k], rtol=1e-10, atol=1e-11, err_msg=k)


def test_finite_differences():
    indptr, indices = random_multigraph(3, 7, 20, undirected=False)
    n = len(indptr) - 1
    Wh, a_l, a_r, g = _inputs(11, n, 2, 3)
    Wh, a_l, a_r, g = (x.astype(np.float64) for x in (Wh, a_l, a_r, g))
    b = og.gat_backward(indptr, indices, Wh, a_l, a_r, g)

    def loss(W, al, ar):
        return float((og.gat_forward(indptr, indices, W, al, ar)["out"] * g).sum())

    h = 1e-6
    rng = np.random.default_rng(0)
    for _ in range(12):
        idx = tuple(rng.integers(s) for s in Wh.shape)
        Wp, Wm = Wh.copy(), Wh.copy()
        Wp[idx] += h; Wm[idx] -= h
        fd = (loss(Wp, a_l, a_r) - loss(Wm, a_l, a_r)) / (2 * h)
        assert abs(fd - b["grad_feat"][idx]) < 1e-7 * max(1.0, abs(fd))
    for which, arr in (("grad_attn_l", a_l), ("grad_attn_r", a_r)):
        for _ in range(4):
            idx = tuple(rng.integers(s) for s in arr.shape)
            p, m = arr.copy(), arr.copy()
            p[idx] += h; m[idx] -= h
            if which == "grad_attn_l":
                fd = (loss(Wh, p, a_r) - loss(Wh, m, a_r)) / (2 * h)
            else:
                fd = (loss(Wh, a_l, p) - loss(Wh, a_l, m)) / (2 * h)
            assert abs(fd - b[which][idx]) < 1e-7 * max(1.0, abs(fd))


def test_softmax_sums_to_one_and_empty_rows():
    indptr, indices = random_multigraph(4, 30, 120, undirected=False, isolated=5)
    n = len(indptr) - 1
    Wh, a_l, a_r, g = _inputs(5, n, 4, 2)
    f = og.gat_forward(indptr, indices, Wh, a_l, a_r)
    deg = np.diff(indptr)
    dst = np.repeat(np.arange(n), deg)
    sums = np.zeros((n, 4))
    np.add.at(sums, dst, f["alpha"])
    np.testing.assert_allclose(sums[deg > 0], 1.0, rtol=0, atol=1e-14)
    assert np.all(f["out"][deg == 0] == 0) and np.all(f["lse"][deg == 0] == -np.inf)
    b = og.gat_backward(indptr, indices, Wh, a_l, a_r, g)
    assert np.all(b["del"][deg == 0] == 0)


@pytest.mark.parametrize("impl_cls", [PyImpl, CImpl], ids=["python", "c"])
def test_zero_attention_is_mean_aggregation(impl_cls):
    """a_l = a_r = 0 -> alpha = 1/deg -> out = D^-1 A Wh (scipy.sparse SpMM)."""
    indptr, indices = random_multigraph(6, 25, 100, undirected=True)
    n = len(indptr) - 1
    Wh, _, _, _ = _inputs(8, n, 3, 4)
    z = np.zeros((3, 4), np.float32)
    f = impl_cls.fwd(indptr, indices, Wh, z, z)
    deg = np.diff(indptr).astype(np.float64)
    A = sp.csr_matrix((np.ones(len(indices)), np.asarray(indices), indptr), shape=(n, n))
    Dinv = sp.diags(np.where(deg > 0, 1.0 / np.maximum(deg, 1), 0.0))
    ref = (Dinv @ A @ Wh.reshape(n, -1).astype(np.float64)).reshape(n, 3, 4)
    np.testing.assert_allclose(f["out"], ref, rtol=1e-13, atol=1e-13)


def test_slope_one_cancels_destination_term():
    """slope = 1: s = el_i + er_j, el_i is constant per softmax row -> out independent of a_l."""
    indptr, indices = random_multigraph(9, 20, 80)
    n = len(indptr) - 1
    Wh, a_l, a_r, _ = _inputs(10, n, 2, 4)
    f1 = og.gat_forward(indptr, indices, Wh, a_l, a_r, slope=1.0)
    f2 = og.gat_forward(indptr, indices, Wh, 3.0 * a_l - 1.0, a_r, slope=1.0)
    np.testing.assert_allclose(f1["out"], f2["out"], rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("impl_cls", [PyImpl, CImpl], ids=["python", "c"])
def test_in_degree_one_copies_source(impl_cls):
    src = [3, 0, 1, 2]
    dst = [0, 1, 2, 3]
    indptr, indices = from_edge_list(5, src, dst)
    Wh, a_l, a_r, _ = _inputs(12, 5, 2, 3)
    f = impl_cls.fwd(indptr, indices, Wh, a_l, a_r)
    for s, d in zip(src, dst):
        assert np.array_equal(f["out"][d], Wh[s].astype(np.float64))


@pytest.mark.parametrize("impl_cls", [PyImpl, CImpl], ids=["python", "c"])
def test_relabelling_equivariance(impl_cls):
    indptr, indices = random_multigraph(13, 40, 200, undirected=False, isolated=3)
    n = len(indptr) - 1
    Wh, a_l, a_r, g = _inputs(14, n, 4, 2)
    perm = np.random.default_rng(1).permutation(n)        # perm[new] = old
    new_of_old = np.empty(n, np.int64); new_of_old[perm] = np.arange(n)
    s_old = np.asarray(indices, np.int64)
    d_old = np.repeat(np.arange(n), np.diff(indptr))
    ip2, ix2 = from_edge_list(n, new_of_old[s_old], new_of_old[d_old])
    f1 = impl_cls.fwd(indptr, indices, Wh, a_l, a_r)
    f2 = impl_cls.fwd(ip2, ix2, Wh[perm], a_l, a_r)
    np.testing.assert_allclose(f2["out"], f1["out"][perm], rtol=1e-13, atol=1e-14)
    b1 = impl_cls.bwd(indptr, indices, Wh, a_l, a_r, g)
    b2 = impl_cls.bwd(ip2, ix2, Wh[perm], a_l, a_r, g[perm])
    np.testing.assert_allclose(b2["grad_feat"], b1["grad_feat"][perm], rtol=1e-12, atol=1e-13)
    np.testing.assert_allclose(b2["grad_attn_l"], b1["grad_attn_l"], rtol=1e-11, atol=1e-12)


def test_backward_invariants():
    indptr, indices = random_multigraph(15, 30, 150, undirected=False)
    n = len(indptr) - 1
    Wh, a_l, a_r, g = _inputs(16, n, 3, 5)
    b = og.gat_backward(indptr, indices, Wh, a_l, a_r, g)
    np.testing.assert_allclose(b["del"].sum(), b["der"].sum(), rtol=1e-12, atol=1e-12)
    # sum over a row's in-edges of ds = alpha (dalpha - Dlt) is 0 (softmax Jacobian rows sum to 0)
    f = og.gat_forward(indptr, indices, Wh, a_l, a_r)
    ds = b["dz"] / np.where(f["z"] > 0, 1.0, og.SLOPE)
    dst = np.repeat(np.arange(n), np.diff(indptr))
    row = np.zeros((n, 3))
    np.add.at(row, dst, ds)
    assert np.max(np.abs(row)) < 1e-12
    # all-equal neighbour rows -> ds = 0 for that row
    Wh2 = Wh.copy()
    i = int(np.argmax(np.diff(indptr)))
    for j in indices[indptr[i]:indptr[i + 1]]:
        Wh2[j] = Wh2[indices[indptr[i]]]
    b2 = og.gat_backward(indptr, indices, Wh2, a_l, a_r, g)
    assert np.max(np.abs(b2["dz"][indptr[i]:indptr[i + 1]])) < 1e-13


def test_golden_tiny():
    case = json.load(open(os.path.join(GOLDEN, "gat_tiny.json")))
    indptr, indices = from_edge_list(case["n"], case["src"], case["dst"])
    Wh = np.asarray(case["Wh"], np.float64).reshape(case["n"], 1, 1)
    one = np.ones((1, 1))
    f = og.gat_forward(indptr, indices, Wh, one, one)
    np.testing.assert_allclose(f["out"][0, 0, 0], case["out0"], rtol=1e-15)
    np.testing.assert_allclose(f["lse"][0, 0], case["lse0"], rtol=1e-15)
    c = coracle.gat_forward(indptr, indices, Wh.astype(np.float32), one, one)
    np.testing.assert_allclose(c["out"][0, 0, 0], case["out0"], rtol=1e-15)


def test_c_oracle_matches_python_on_bf16_values():
    indptr, indices = random_multigraph(17, 60, 400, undirected=True)
    n = len(indptr) - 1
    Wh, a_l, a_r, g = _inputs(18, n, 4, 8)
    Wh = bf16_round(Wh); g = bf16_round(g)
    p = og.gat_backward(indptr, indices, Wh, a_l, a_r, g)
    c = coracle.gat_backward(indptr, indices, Wh, a_l, a_r, g)
    for k in ("grad_feat", "grad_attn_l", "grad_attn_r", "del", "der"):
        np.testing.assert_allclose(c[k], p[k], rtol=1e-12, atol=1e-12, err_msg=k)
    rows = np.array([0, 5, n - 1])
    r = coracle.gat_forward_rows(indptr, indices, Wh, a_l, a_r, rows)
    pf = og.gat_forward(indptr, indices, Wh, a_l, a_r)
    np.testing.assert_allclose(r["out"], pf["out"][rows], rtol=1e-13, atol=1e-14)
    srcs = np.array([1, 7, n - 2])
    gs = coracle.gat_backward_srcs(indptr, indices, Wh, a_l, a_r, g, srcs)
    np.testing.assert_allclose(gs, p["grad_feat"][srcs], rtol=1e-11, atol=1e-12)


def test_projection():
    rng = np.random.default_rng(3)
    x = rng.standard_normal((13, 7)); w = rng.standard_normal((7, 6)); gf = rng.standard_normal((13, 6))
    wh = og.project_forward(x, w)
    ref = np.einsum("nk,kd->nd", x, w)
    np.testing.assert_allclose(wh, ref, rtol=1e-13)
    xt = torch.tensor(x, requires_grad=True); wt = torch.tensor(w, requires_grad=True)
    (xt @ wt * torch.tensor(gf)).sum().backward()
    b = og.project_backward(x, w, gf)
    np.testing.assert_allclose(b["grad_w"], wt.grad.numpy(), rtol=1e-12)
    np.testing.assert_allclose(b["grad_x"], xt.grad.numpy(), rtol=1e-12)
