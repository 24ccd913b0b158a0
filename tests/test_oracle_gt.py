"""Pins for oracle/gt.py (Graph Transformer attention),
against formulations that share none of its code:

* dense masked attention (per head, an [n, n] logit matrix with log-multiplicity
  bias so duplicate edges count as separate softmax terms) through torch's
  softmax and matmul, and its gradients by torch autograd (fp64);
* K = 0 makes every score equal, so out_i is the plain mean of V over the
  in-edge multiset of i;
* a single in-edge gives alpha = 1 and out_i = V_j exactly.
"""
import numpy as np
import pytest
import torch

from oracle import gt
from synth.tiny import random_multigraph, to_edge_list


def _qkvg(seed, n, H, F):
    rng = np.random.default_rng(seed)
    return [rng.standard_normal((n, H, F)) for _ in range(4)]


def _dense(ip, ix, Q, K, V, g):
    n, H, F = Q.shape
    src, dst = to_edge_list(ip, ix)
    C = np.zeros((n, n))
    np.add.at(C, (dst, src), 1.0)
    has = torch.tensor(C.sum(1) > 0)
    bias = torch.tensor(np.where(C > 0, np.log(np.where(C > 0, C, 1.0)), -np.inf))
    q, k, v = (torch.tensor(a, dtype=torch.float64, requires_grad=True) for a in (Q, K, V))
    logits = torch.einsum("ihf,jhf->hij", q, k) / np.sqrt(F) + bias
    logits = torch.where(has[None, :, None], logits, torch.zeros_like(logits))
    att = torch.softmax(logits, dim=-1) * has[None, :, None]
    out = torch.einsum("hij,jhf->ihf", att, v)
    lse = torch.where(has[None], torch.logsumexp(logits, -1), torch.full_like(logits[..., 0], -np.inf)).T
    (out * torch.tensor(g)).sum().backward()
    return {"out": out.detach().numpy(), "lse": lse.detach().numpy(), "grad_q": q.grad.numpy(),
            "grad_k": k.grad.numpy(), "grad_v": v.grad.numpy()}


@pytest.mark.parametrize("seed", range(4))
def test_gt_vs_dense_autograd(seed):
    n = 40 + 13 * seed
    ip, ix = random_multigraph(seed, n, 6 * n, undirected=bool(seed % 2), isolated=3)
    H, F = (1, 4, 2, 8)[seed], (8, 16, 4, 32)[seed]
    Q, K, V, g = _qkvg(seed, n, H, F)
    f = gt.gt_forward(ip, ix, Q, K, V)
    b = gt.gt_backward(ip, ix, Q, K, V, g, fwd=f)
    d = _dense(ip, ix, Q, K, V, g)
    np.testing.assert_allclose(f["out"], d["out"], rtol=1e-11, atol=1e-12)
    np.testing.assert_array_equal(np.isfinite(f["lse"]), np.isfinite(d["lse"]))
    fin = np.isfinite(f["lse"])
    np.testing.assert_allclose(f["lse"][fin], d["lse"][fin], rtol=1e-11, atol=1e-12)
    for k in ("grad_q", "grad_k", "grad_v"):
        np.testing.assert_allclose(b[k], d[k], rtol=1e-10, atol=1e-11, err_msg=k)


def test_gt_zero_keys_is_multiset_mean():
    ip, ix = random_multigraph(7, 60, 400, isolated=5)
    Q, _, V, _ = _qkvg(1, 60, 2, 8)
    f = gt.gt_forward(ip, ix, Q, np.zeros_like(Q), V)
    for i in range(60):
        js = ix[ip[i]:ip[i + 1]]
        want = V[js].mean(0) if len(js) else np.zeros((2, 8))
        np.testing.assert_allclose(f["out"][i], want, rtol=1e-12, atol=1e-13)


def test_gt_single_in_edge_is_exact_copy():
    ip = np.array([0, 1, 2, 2], np.int64)
    ix = np.array([2, 0], np.int32)
    Q, K, V, g = _qkvg(3, 3, 2, 4)
    f = gt.gt_forward(ip, ix, Q, K, V)
    assert np.array_equal(f["out"][0], V[2]) and np.array_equal(f["out"][1], V[0])
    assert np.all(f["out"][2] == 0) and np.all(np.isneginf(f["lse"][2]))
    b = gt.gt_backward(ip, ix, Q, K, V, g, fwd=f)
    assert np.all(b["grad_q"] == 0) and np.all(b["grad_k"] == 0)   # alpha = 1 regardless of the score
    assert np.array_equal(b["grad_v"][2], g[0]) and np.array_equal(b["grad_v"][0], g[1])
