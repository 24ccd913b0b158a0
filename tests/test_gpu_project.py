"""GPU parity of the projection GEMMs (rows a2 / a9) against fp64 numpy.

bf16 mode runs the hand-written tcgen05 kernels (csrc/umma_gemm.cu): TMA-staged
operands, tcgen05.mma with the fp32 accumulator in TMEM, el/er computed in the
forward GEMM's epilogue from the stored bf16 Wh.  Shapes cover every operand
layout the layer uses (K-major and MN-major A/B), ragged row counts (not a
multiple of the 128-row tile), K not a multiple of the 64-wide K block
(in_dim = 100 inside ldx = 104, as products' first layer), D = 64 / 256 / 512
(one and two column tiles), and the dW split over rows with its fixed-order
reduction (above 8 K blocks of rows) or unsplit, written directly (up to 8).  Bars: Wh and dX elementwise within bf16 rounding of the fp64 value
(2^-8 |ref|) plus fp32-accumulation noise; el/er, dW normwise 1e-4 max|ref|
beyond the rounding they inherit (north_star's bf16 bar is 2e-2 per tensor;
these are tighter because a GEMM has no exp/log chain).
"""
import numpy as np
import pytest
import torch

import synth
from paper_conf_icdcs_dengr24_b200 import mega as M

pytestmark = pytest.mark.gpu

SHAPES = [  # rows, in_dim, ldx, heads, head_dim
    (1000, 100, 104, 4, 128),    # products layer 1 (K tail inside the padded row)
    (777, 512, 512, 4, 128),     # products hidden
    (2049, 608, 608, 4, 64),     # reddit (5 K blocks, last one partial), D = 256
    (300, 128, 128, 8, 8),       # cora/pubmed-like D = 64, head_dim 8
    (129, 1440, 1440, 8, 8),     # cora's F_in
    (5000, 128, 128, 8, 16),     # the batch workloads' hidden layer
    (64, 64, 64, 1, 64),         # one partial row tile (dW unsplit, written directly)
    (500, 128, 128, 8, 16),      # dW unsplit (<= 8 K blocks)
    (20000, 512, 512, 4, 128),   # dW split over rows + fixed-order reduction
]


def _bf(a):
    return synth.bf16_round(np.asarray(a, np.float32))


@pytest.mark.parametrize("rows,in_dim,ldx,H,F", SHAPES)
def test_projection_tcgen05(cuda_device, rows, in_dim, ldx, H, F):
    rng = np.random.default_rng(rows + in_dim)
    D = H * F
    x = np.zeros((rows, ldx), np.float32)
    x[:, :in_dim] = _bf(rng.standard_normal((rows, in_dim)))
    w = _bf(rng.uniform(-0.1, 0.1, (in_dim, D)))
    a_l = (rng.standard_normal(D) / np.sqrt(F)).astype(np.float32)
    a_r = (rng.standard_normal(D) / np.sqrt(F)).astype(np.float32)
    gf = _bf(rng.standard_normal((rows, D)))
    dev = "cuda"
    xt = torch.tensor(x, device=dev).bfloat16()
    wt = torch.tensor(w, device=dev).bfloat16()
    feat = torch.full((rows, D), float("nan"), device=dev).bfloat16()
    ctx = torch.zeros(M.MEGA_CTX_PLANES, rows, H, device=dev)
    M.mega_project_fwd(xt, wt, torch.tensor(a_l, device=dev), torch.tensor(a_r, device=dev), H, F, feat, ctx, rows,
                       in_dim=in_dim)
    gft = torch.tensor(gf, device=dev).bfloat16()
    gw = torch.full((in_dim, D), float("nan"), device=dev)
    gx = torch.full((rows, ldx), float("nan"), device=dev).bfloat16()
    ws = torch.empty(max(256, M.mega_project_workspace_bytes(rows, in_dim, H, F, M.MEGA_BF16)), dtype=torch.uint8,
                     device=dev)
    M.mega_project_bwd(xt, wt, H, F, gft, gw, gx, in_dim=in_dim, ws=ws)
    torch.cuda.synchronize()
    X = x[:, :in_dim].astype(np.float64)
    W = w.astype(np.float64)
    # ---- forward: Wh and the el/er epilogue ----
    ref = X @ W
    got = feat.float().cpu().numpy()
    scale = np.abs(ref).max()
    assert np.all(np.abs(got - ref) <= 2.0 ** -8 * np.abs(ref) + 1e-5 * scale), "Wh"
    whb = got.reshape(rows, H, F).astype(np.float64)          # el/er are computed from the stored bf16 Wh
    el = np.einsum("nhf,hf->nh", whb, a_l.reshape(H, F))
    er = np.einsum("nhf,hf->nh", whb, a_r.reshape(H, F))
    for name, g_, r_ in (("el", ctx[0].cpu().numpy(), el), ("er", ctx[1].cpu().numpy(), er)):
        assert np.max(np.abs(g_ - r_)) <= 1e-4 * np.abs(r_).max() + 1e-6, name
    # ---- backward: dW (fp32) and dX (bf16, padding columns zero) ----
    G = gf.astype(np.float64)
    dw = X.T @ G
    assert np.max(np.abs(gw.cpu().numpy() - dw)) <= 1e-4 * np.abs(dw).max(), "dW"
    dx = G @ W.T
    gxn = gx.float().cpu().numpy()
    assert np.all(np.abs(gxn[:, :in_dim] - dx) <= 2.0 ** -8 * np.abs(dx) + 1e-5 * np.abs(dx).max()), "dX"
    pad = (in_dim + 7) // 8 * 8
    assert np.all(gxn[:, in_dim:pad] == 0), "dX padding columns"


def test_projection_deterministic(cuda_device):
    rows, in_dim, H, F = 30000, 512, 4, 128
    rng = np.random.default_rng(1)
    D = H * F
    xt = torch.tensor(_bf(rng.standard_normal((rows, in_dim))), device="cuda").bfloat16()
    wt = torch.tensor(_bf(rng.uniform(-0.1, 0.1, (in_dim, D))), device="cuda").bfloat16()
    gft = torch.tensor(_bf(rng.standard_normal((rows, D))), device="cuda").bfloat16()
    ws = torch.empty(M.mega_project_workspace_bytes(rows, in_dim, H, F, M.MEGA_BF16), dtype=torch.uint8,
                     device="cuda")
    outs = []
    for _ in range(2):
        gw = torch.empty(in_dim, D, device="cuda")
        M.mega_project_bwd(xt, wt, H, F, gft, gw, None, in_dim=in_dim, ws=ws)
        outs.append(gw.clone())
    assert torch.equal(outs[0], outs[1])
