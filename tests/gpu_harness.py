"""Shared driver for the GPU parity tests: run the product (libmega.so via the
binding) and the oracle on the same seeded inputs, in old node ids."""
from __future__ import annotations

import numpy as np
import torch

import synth
from paper_conf_icdcs_dengr24_b200 import mega as M
from paper_conf_icdcs_dengr24_b200.layer import GATLayer

DT = {"fp32": torch.float32, "bf16": torch.bfloat16}


def inputs(seed, n, H, F, bf16):
    rng = np.random.default_rng(seed)
    Wh = rng.standard_normal((n, H, F)).astype(np.float32)
    a_l = (rng.standard_normal((H, F)) / np.sqrt(F)).astype(np.float32)
    a_r = (rng.standard_normal((H, F)) / np.sqrt(F)).astype(np.float32)
    g = rng.standard_normal((n, H, F)).astype(np.float32)
    if bf16:
        Wh, g = synth.bf16_round(Wh), synth.bf16_round(g)
    return Wh, a_l, a_r, g


def run_attention(layout, Wh_old, a_l, a_r, g_old, dtype, slope=M.SLOPE, parts=None, dev="cuda"):
    """mega_gat_fwd + mega_gat_bwd on every part of `layout` (parts run one after
    another on this GPU; partial grad_feat of the source phase is summed over
    parts before the destination phase, as the k-GPU reduce-scatter does).
    Returns old-order numpy arrays."""
    n, H, F = Wh_old.shape
    D = H * F
    v0 = layout.view(0)
    perm = v0["perm"].astype(np.int64)
    k = v0["num_parts"]
    tdt = DT[dtype]
    feat = torch.tensor(Wh_old.reshape(n, D)[perm], dtype=torch.float32, device=dev).to(tdt).contiguous()
    g_new = torch.tensor(g_old.reshape(n, D)[perm], dtype=torch.float32, device=dev).to(tdt).contiguous()
    al = torch.tensor(a_l.reshape(-1), device=dev)
    ar = torch.tensor(a_r.reshape(-1), device=dev)
    ctx = torch.zeros(M.MEGA_CTX_PLANES, n, H, dtype=torch.float32, device=dev)
    out_full = torch.empty(n, D, dtype=tdt, device=dev)
    gal = torch.zeros(D, device=dev)
    gar = torch.zeros(D, device=dev)
    part_ids = range(k) if parts is None else parts
    states = []
    for p in part_ids:
        layout.bind(p)
        v = layout.view(p, arrays=False)
        b0, b1 = v["row_begin"], v["row_end"]
        fws, bws = M.mega_gat_workspace_bytes(layout, p, H, F, M._dtype_code(feat))
        wsf = torch.empty(max(fws, 256), dtype=torch.uint8, device=dev)
        wsb = torch.empty(max(bws, 256), dtype=torch.uint8, device=dev)
        out = out_full[b0:b1]
        M.mega_gat_fwd(layout, p, feat, al, ar, H, F, out, ctx, wsf, negative_slope=slope)
        states.append((p, b0, b1, wsb))
    # source phase per part -> partial grad_feat and der plane; sum over parts (the k-GPU
    # reduce-scatter), then the destination phase per part on its own rows
    partial, der_parts = [], []
    for p, b0, b1, wsb in states:
        gf = torch.zeros(n, D, dtype=torch.float32, device=dev)
        M.mega_gat_bwd(layout, p, feat, al, ar, H, F, out_full[b0:b1], g_new[b0:b1], ctx, gf,
                       torch.zeros(D, device=dev), torch.zeros(D, device=dev), wsb, negative_slope=slope,
                       flags=M.MEGA_BWD_PHASE_SRC)
        partial.append(gf)
        der_parts.append(ctx[4].clone())
    gfeat = torch.stack(partial).sum(0)
    ctx[4] = torch.stack(der_parts).sum(0)
    for p, b0, b1, wsb in states:
        tmp_l = torch.zeros(D, device=dev)
        tmp_r = torch.zeros(D, device=dev)
        M.mega_gat_bwd(layout, p, feat, al, ar, H, F, out_full[b0:b1], g_new[b0:b1], ctx, gfeat, tmp_l, tmp_r,
                       wsb, negative_slope=slope, flags=M.MEGA_BWD_PHASE_DST)
        gal += tmp_l
        gar += tmp_r
    if k == 1:   # the single-call path (both phases) must agree with the split one
        gf1 = torch.zeros(n, D, dtype=torch.float32, device=dev)
        l1, r1 = torch.zeros(D, device=dev), torch.zeros(D, device=dev)
        p, b0, b1, wsb = states[0]
        M.mega_gat_bwd(layout, p, feat, al, ar, H, F, out_full[b0:b1], g_new[b0:b1], ctx, gf1, l1, r1, wsb,
                       negative_slope=slope)
        assert torch.equal(gf1, gfeat) and torch.equal(l1, gal) and torch.equal(r1, gar)
    torch.cuda.synchronize()
    inv = np.empty(n, np.int64)
    inv[perm] = np.arange(n)

    def old(t, shape):
        a = t.float().cpu().numpy()
        return a[inv].reshape(shape)

    return {"out": old(out_full, (n, H, F)), "lse": old(ctx[2], (n, H)), "el": old(ctx[0], (n, H)),
            "er": old(ctx[1], (n, H)), "grad_feat": old(gfeat, (n, H, F)),
            "grad_attn_l": gal.cpu().numpy().reshape(H, F), "grad_attn_r": gar.cpu().numpy().reshape(H, F)}


def assert_fp32_close(got, ref, name):
    """north_star fp32 bar: |gpu - ref| <= 1e-4 + 1e-5 |ref| elementwise."""
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    fin = np.isfinite(ref)
    assert np.array_equal(fin, np.isfinite(got)), f"{name}: finiteness differs"
    assert np.all(got[~fin] == ref[~fin]), f"{name}: infinities differ"
    err = np.abs(got[fin] - ref[fin])
    tol = 1e-4 + 1e-5 * np.abs(ref[fin])
    bad = err > tol
    assert not bad.any(), f"{name}: {bad.sum()} elements out of tolerance, max err {err.max():.3e}"


def assert_bf16_close(got, ref, name, extra=None):
    """north_star bf16 bar: max|gpu - ref| <= 2e-2 max|ref| per tensor.
    `extra` (elementwise, optional) adds a derived error bound (see dlt_bf16_bound)."""
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    fin = np.isfinite(ref)
    assert np.array_equal(fin, np.isfinite(got)), f"{name}: finiteness differs"
    scale = np.max(np.abs(ref[fin])) if fin.any() else 0.0
    err = np.abs(got[fin] - ref[fin])
    tol = 2e-2 * scale + (0.0 if extra is None else np.asarray(extra, np.float64).reshape(ref.shape)[fin])
    bad = err > tol
    assert not bad.any(), (f"{name}: {bad.sum()} elements out of tolerance, max err {err.max():.3e} "
                           f"(2e-2 * {scale:.3e}{'' if extra is None else ' + derived bound'})")


def dlt_bf16_bound(ip, ix, Wh, a_l, a_r, g, slope=M.SLOPE):
    """Elementwise bound on the grad_attn_l / grad_attn_r error that bf16 storage of
    `out` introduces (DESIGN.md R-prec, "Dlt bound").  The GPU forms Dlt_i = g_i . out_i
    from the STORED bf16 out (a6 saves an edge pass that way), so its grad_attn carry
    the effect of that rounding, which does not vanish where the exact result is 0 by
    cancellation.  The bound has three parts, all computed from the fp64 oracle
    (never from the GPU):
      1. the exact effect of rounding out to bf16: |da(Dlt from bf16(out)) - da(exact)|;
      2. elements of out within 2^-16 relative of a bf16 rounding midpoint may round the
         other way on the GPU (its fp32 out differs from the exact one by ~2^-20
         relative): each costs at most one bf16 ulp, |g_i,f| ulp(out_i,f), in Dlt_i;
      3. the two F-term fp32 dot products (dalpha_e = g_i . Wh_j, Dlt_i):
         F 2^-23 (A_i + B_e), A_i = sum_f |g_i||out_i|, B_e = sum_f |g_i||Wh_j|.
    Parts 2-3 give eps_e per edge and head; dz_e = alpha_e (dalpha_e - Dlt_i) lf_e with
    lf_e <= 1 gives |d del_i| <= sum_In alpha eps, |d der_j| <= sum_Out alpha eps and
    |d da_l[h,f]| <= sum_i |d del_i,h| |Wh_i,h,f| (da_r likewise with der)."""
    import synth as _synth
    from oracle import gat as og
    Wh = np.asarray(Wh, np.float64)
    g = np.asarray(g, np.float64)
    n, H, F = Wh.shape
    f = og.gat_forward(ip, ix, Wh, a_l, a_r, slope)
    b = og.gat_backward(ip, ix, Wh, a_l, a_r, g, slope, fwd=f)
    out = f["out"]
    outb = _synth.bf16_round(out.astype(np.float32)).astype(np.float64)
    b_r = og.gat_backward(ip, ix, Wh, a_l, a_r, g, slope, fwd={**f, "out": outb})     # part 1
    # part 2: distance to the nearest bf16 rounding midpoint, relative
    ulp = np.where(out != 0, 2.0 ** (np.floor(np.log2(np.abs(np.where(out != 0, out, 1.0)))) - 7), 0.0)
    mid_dist = np.abs(np.abs(out - outb) - 0.5 * ulp)
    near = mid_dist <= 2.0 ** -16 * np.abs(out)
    flip = np.einsum("nhf,nhf->nh", np.abs(g), np.where(near, ulp, 0.0))
    deg = np.diff(np.asarray(ip, np.int64))
    dst = np.repeat(np.arange(n), deg)
    src = np.asarray(ix, np.int64)
    A = np.einsum("nhf,nhf->nh", np.abs(g), np.abs(out))
    B = np.einsum("ehf,ehf->eh", np.abs(g[dst]), np.abs(Wh[src]))
    eps = flip[dst] + F * 2.0 ** -23 * (A[dst] + B)                                 # parts 2 + 3
    t = f["alpha"] * eps
    ddel = np.zeros((n, H))
    np.add.at(ddel, dst, t)
    dder = np.zeros((n, H))
    np.add.at(dder, src, t)
    aW = np.abs(Wh)
    return {"grad_attn_l": np.abs(b_r["grad_attn_l"] - b["grad_attn_l"]) + np.einsum("nh,nhf->hf", ddel, aW),
            "grad_attn_r": np.abs(b_r["grad_attn_r"] - b["grad_attn_r"]) + np.einsum("nh,nhf->hf", dder, aW)}


def assert_fp32_close_reduction(got, ref, name):
    """fp32 bar for the parameter gradients (DESIGN.md R-tol): they are sums over all N
    rows of terms whose own fp32 relative error is ~1e-6 (exp/log chains), so the
    relative part is taken against the tensor's scale: |d| <= 1e-4 + 1e-5 max|ref|
    (tests/test_tolerance_fp32.py shows the elementwise form is out of reach for fp32)."""
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    err = np.abs(got - ref)
    tol = 1e-4 + 1e-5 * np.max(np.abs(ref))
    assert np.all(err <= tol), f"{name}: max err {err.max():.3e} > {tol:.3e}"


REDUCTIONS = ("grad_attn_l", "grad_attn_r", "grad_w")


def check(got, ref, dtype, keys=("out", "lse", "grad_feat", "grad_attn_l", "grad_attn_r"), graph=None):
    """graph = (indptr, indices, Wh, a_l, a_r, g) in old ids: in bf16 mode the attention-parameter
    gradients then also get the derived Dlt bound (dlt_bf16_bound)."""
    bound = dlt_bf16_bound(*graph) if (graph is not None and dtype == "bf16") else {}
    for k in keys:
        if dtype == "fp32":
            (assert_fp32_close_reduction if k in REDUCTIONS else assert_fp32_close)(got[k], ref[k], k)
        else:
            assert_bf16_close(got[k], ref[k], k, extra=bound.get(k))


def layer(layout, x_new, w, a_l, a_r, H, F, dtype, want_grad_x=True):
    tdt = DT[dtype]
    dev = "cuda"
    xt = torch.tensor(x_new, device=dev).to(tdt).contiguous()
    wt = torch.tensor(w, device=dev).to(tdt).contiguous()
    L = GATLayer(layout, xt, wt, torch.tensor(a_l, device=dev), torch.tensor(a_r, device=dev), H, F,
                 want_grad_x=want_grad_x)
    return L
