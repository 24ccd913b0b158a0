"""GAT attention over a graph, fp64, per edge — the plain definition.

Test infrastructure only (see oracle/__init__.py).

The layer skeleton is PAPER.md:51 (§II-A): h'_u = func(w, h_u,
aggregate_{v in N(u)}(h_v, e_{v,u})), i.e. a graph operator that scatters node
values to edges and gathers them back (Fig. 2) followed by a
neural operator.  The attention function is GAT [14] (cited at PAPER.md:49) as
BASELINE.json's north_star writes it:

    e_ij  = LeakyReLU(a_l . Wh_i + a_r . Wh_j)          i = destination, j = source
    alpha = softmax over the in-edges of i
    out_i = sum_e alpha_e Wh_j

with the readings of DESIGN.md §"Readings of the paper": slope = (double)0.2f,
derivative slope at z <= 0 (R3); no self-loops added, duplicates are separate
softmax terms (R4, R5); zero in-degree -> out = 0, lse = -inf (R6); heads
concatenated, no bias/activation (R7).

Graph arguments are CSR by destination: indptr int64 [n+1], indices [m]
(source ids).  Feature arrays are float64 [n, H, F]; a_l/a_r are [H, F].
"""
from __future__ import annotations

import numpy as np

SLOPE = float(np.float32(0.2))  # (double)0.2f, reading R3
_CHUNK = 1 << 18


def _edges(indptr, indices):
    deg = np.diff(np.asarray(indptr, dtype=np.int64))
    dst = np.repeat(np.arange(len(deg), dtype=np.int64), deg)
    return np.asarray(indices, dtype=np.int64), dst


def attention_halves(Wh, a_l, a_r):
    """el_i = sum_f a_l[h,f] Wh[i,h,f] (destination term), er_j likewise with a_r
    (source term) — north_star's e_ij split into its two node terms."""
    Wh = np.asarray(Wh, dtype=np.float64)
    return (np.einsum("nhf,hf->nh", Wh, np.asarray(a_l, np.float64)),
            np.einsum("nhf,hf->nh", Wh, np.asarray(a_r, np.float64)))


def scores(el, er, src, dst, slope=SLOPE):
    """z_e = el_dst + er_src; s_e = LeakyReLU(z_e)   (north_star e_ij)."""
    z = el[dst] + er[src]
    return z, np.where(z > 0, z, slope * z)


def gat_forward(indptr, indices, Wh, a_l, a_r, slope=SLOPE):
    """Two-pass edge softmax and aggregation.

    Returns dict(out [n,H,F], lse [n,H], el, er [n,H], alpha [m,H]).
    """
    Wh = np.asarray(Wh, dtype=np.float64)
    n, H, F = Wh.shape
    src, dst = _edges(indptr, indices)
    el, er = attention_halves(Wh, a_l, a_r)
    z, s = scores(el, er, src, dst, slope)
    m = np.full((n, H), -np.inf)
    np.maximum.at(m, dst, s)                       # m_i = max_e s_e
    p = np.exp(s - m[dst])
    S = np.zeros((n, H))
    np.add.at(S, dst, p)                           # S_i = sum_e exp(s_e - m_i)
    alpha = p / S[dst]                             # alpha_e
    out = np.zeros((n, H, F))
    for b in range(0, len(src), _CHUNK):           # out_i = sum_e alpha_e Wh_j
        sl = slice(b, b + _CHUNK)
        np.add.at(out, dst[sl], alpha[sl, :, None] * Wh[src[sl]])
    with np.errstate(divide="ignore"):
        lse = np.where(S > 0, m + np.log(np.where(S > 0, S, 1.0)), -np.inf)
    return {"out": out, "lse": lse, "el": el, "er": er, "alpha": alpha, "z": z}


def gat_backward(indptr, indices, Wh, a_l, a_r, grad_out, slope=SLOPE, fwd=None):
    """Closed-form backward of gat_forward:

        dalpha_e = g_i . Wh_j            Dlt_i = g_i . out_i
        ds_e = alpha_e (dalpha_e - Dlt_i)     dz_e = ds_e * (z_e > 0 ? 1 : slope)
        del_i = sum_{e in In(i)} dz_e    der_j = sum_{e in Out(j)} dz_e
        dWh_j = sum_{e=(j->i)} alpha_e g_i + der_j a_r + del_j a_l
        da_l = sum_i del_i Wh_i          da_r = sum_j der_j Wh_j
    """
    Wh = np.asarray(Wh, dtype=np.float64)
    g = np.asarray(grad_out, dtype=np.float64)
    a_l = np.asarray(a_l, np.float64)
    a_r = np.asarray(a_r, np.float64)
    n, H, F = Wh.shape
    if fwd is None:
        fwd = gat_forward(indptr, indices, Wh, a_l, a_r, slope)
    src, dst = _edges(indptr, indices)
    alpha, z, out = fwd["alpha"], fwd["z"], fwd["out"]
    Dlt = np.einsum("nhf,nhf->nh", g, out)
    dWh = np.zeros((n, H, F))
    dz = np.empty((len(src), H))
    for b in range(0, len(src), _CHUNK):
        sl = slice(b, b + _CHUNK)
        dalpha = np.einsum("ehf,ehf->eh", g[dst[sl]], Wh[src[sl]])
        ds = alpha[sl] * (dalpha - Dlt[dst[sl]])
        dz[sl] = ds * np.where(z[sl] > 0, 1.0, slope)
        np.add.at(dWh, src[sl], alpha[sl, :, None] * g[dst[sl]])
    dl = np.zeros((n, H))
    np.add.at(dl, dst, dz)
    dr = np.zeros((n, H))
    np.add.at(dr, src, dz)
    dWh += dr[:, :, None] * a_r[None] + dl[:, :, None] * a_l[None]
    return {"grad_feat": dWh, "grad_attn_l": np.einsum("nh,nhf->hf", dl, Wh),
            "grad_attn_r": np.einsum("nh,nhf->hf", dr, Wh), "del": dl, "der": dr, "Dlt": Dlt, "dz": dz}


def project_forward(x, w):
    """Linear projection Wh = X W (the neural operator), fp64."""
    return np.asarray(x, np.float64) @ np.asarray(w, np.float64)


def project_backward(x, w, grad_feat):
    """dW = X^T dWh, dX = dWh W^T (last line)."""
    x = np.asarray(x, np.float64)
    gf = np.asarray(grad_feat, np.float64)
    return {"grad_w": x.T @ gf, "grad_x": gf @ np.asarray(w, np.float64).T}
