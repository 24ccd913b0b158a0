"""Graph Transformer attention over a graph, fp64, per edge — the plain definition
(SURVEY.md §8(f) NEXT-3).  The CUDA path it checks is csrc/gt_kernels.cu
(mega_gt_fwd / mega_gt_bwd), compared against this file in tests/test_gpu_gt.py.

Test infrastructure only (see oracle/__init__.py).

The paper's headline model is GT [18] ("adopts the mechanism from
the transformer for computing graph attention coefficients", multi-head; Table
I: extra query/key graph operations).  Its attention module,
restricted to the graph as PAPER.md:51 restricts every aggregation to N(i):

    s_e   = (Q_i . K_j) / sqrt(F)        per head, e = (j -> i), i = destination
    alpha = softmax of s over the in-edges of i
    out_i = sum_e alpha_e V_j

Readings (DESIGN.md R-gt): no score clamp (the public GT code clamps to
[-5, 5]; the paper states no clamp), duplicates are separate softmax terms and
zero in-degree gives out = 0, lse = -inf, as for GAT (R4-R6).  Q, K, V are
float64 [n, H, F]; graph is CSR by destination.
"""
from __future__ import annotations

import numpy as np

from oracle.gat import _edges


def gt_forward(indptr, indices, Q, K, V):
    """Two-pass edge softmax and aggregation.  -> dict(out, lse, alpha, s)."""
    Q, K, V = (np.asarray(a, np.float64) for a in (Q, K, V))
    n, H, F = Q.shape
    src, dst = _edges(indptr, indices)
    s = np.einsum("ehf,ehf->eh", Q[dst], K[src]) / np.sqrt(F)     # s_e
    m = np.full((n, H), -np.inf)
    np.maximum.at(m, dst, s)
    p = np.exp(s - m[dst])
    S = np.zeros((n, H))
    np.add.at(S, dst, p)
    alpha = p / S[dst]
    out = np.zeros((n, H, F))
    np.add.at(out, dst, alpha[:, :, None] * V[src])                # out_i = sum_e alpha_e V_j
    with np.errstate(divide="ignore"):
        lse = np.where(S > 0, m + np.log(np.where(S > 0, S, 1.0)), -np.inf)
    return {"out": out, "lse": lse, "alpha": alpha, "s": s}


def gt_backward(indptr, indices, Q, K, V, grad_out, fwd=None):
    """Closed-form backward of gt_forward:

        dalpha_e = g_i . V_j          Dlt_i = g_i . out_i
        ds_e = alpha_e (dalpha_e - Dlt_i)
        dQ_i = sum_{e in In(i)} ds_e K_j / sqrt(F)
        dK_j = sum_{e in Out(j)} ds_e Q_i / sqrt(F)
        dV_j = sum_{e in Out(j)} alpha_e g_i
    """
    Q, K, V = (np.asarray(a, np.float64) for a in (Q, K, V))
    g = np.asarray(grad_out, np.float64)
    n, H, F = Q.shape
    if fwd is None:
        fwd = gt_forward(indptr, indices, Q, K, V)
    src, dst = _edges(indptr, indices)
    alpha, out = fwd["alpha"], fwd["out"]
    Dlt = np.einsum("nhf,nhf->nh", g, out)
    dalpha = np.einsum("ehf,ehf->eh", g[dst], V[src])
    ds = alpha * (dalpha - Dlt[dst])
    dQ = np.zeros((n, H, F))
    dK = np.zeros((n, H, F))
    dV = np.zeros((n, H, F))
    np.add.at(dQ, dst, ds[:, :, None] * K[src] / np.sqrt(F))
    np.add.at(dK, src, ds[:, :, None] * Q[dst] / np.sqrt(F))
    np.add.at(dV, src, alpha[:, :, None] * g[dst])
    return {"grad_q": dQ, "grad_k": dK, "grad_v": dV, "Dlt": Dlt, "ds": ds}
