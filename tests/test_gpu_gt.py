"""GPU parity of the Graph Transformer edge attention (NEXT-3: mega_gt_fwd /
mega_gt_bwd through the C ABI) against the fp64 oracle oracle/gt.py, element by
element in old node ids.  fp32 mode: |d| <= 1e-4 + 1e-5 |ref| (north_star);
bf16 mode (row-vector kernels over the layout's work items, split rows merged):
max|d| <= 2e-2 max|ref| per tensor, the oracle fed the bf16-rounded Q, K, V and
grad_out the GPU reads (DESIGN.md R-prec)."""
import numpy as np
import pytest
import torch

import synth
from oracle import gt as ogt
from paper_conf_icdcs_dengr24_b200 import mega as M
from tests import gpu_harness as hz

pytestmark = pytest.mark.gpu


def _run(lay, Q, K, V, g, dtype="fp32"):
    """All parts of `lay` on this GPU; grad_k/grad_v partials summed over parts."""
    n, H, F = Q.shape
    D = H * F
    v0 = lay.view(0)
    perm = v0["perm"].astype(np.int64)
    dev = "cuda"
    tdt = hz.DT[dtype]
    t = lambda a: torch.tensor(a.reshape(n, D)[perm], dtype=torch.float32, device=dev).to(tdt).contiguous()
    q, k, v, gn = t(Q), t(K), t(V), t(g)
    out = torch.empty(n, D, device=dev, dtype=tdt)
    lse = torch.empty(n, H, device=dev)
    gq = torch.empty(n, D, device=dev)
    gk = torch.zeros(n, D, device=dev)
    gv = torch.zeros(n, D, device=dev)
    for p in range(v0["num_parts"]):
        lay.bind(p)
        vp = lay.view(p, arrays=False)
        b0, b1 = vp["row_begin"], vp["row_end"]
        ws = torch.empty(max(256, M.mega_gt_workspace_bytes(lay, p, H, F, M._dtype_code(q))), dtype=torch.uint8,
                         device=dev)
        M.mega_gt_fwd(lay, p, q, k, v, H, F, out[b0:b1], lse[b0:b1], ws)
        pk, pv = torch.empty(n, D, device=dev), torch.empty(n, D, device=dev)
        M.mega_gt_bwd(lay, p, q, k, v, H, F, out[b0:b1], lse[b0:b1], gn[b0:b1], gq[b0:b1], pk, pv, ws)
        gk += pk
        gv += pv
    torch.cuda.synchronize()
    inv = np.empty(n, np.int64)
    inv[perm] = np.arange(n)
    o = lambda x, shape: x.float().cpu().numpy()[inv].reshape(shape)
    return {"out": o(out, (n, H, F)), "lse": o(lse, (n, H)), "grad_q": o(gq, (n, H, F)),
            "grad_k": o(gk, (n, H, F)), "grad_v": o(gv, (n, H, F))}


def _check(ip, ix, H, F, seed, parts=1, dtype="fp32", seg=0):
    n = len(ip) - 1
    rng = np.random.default_rng(seed)
    Q, K, V, g = [rng.standard_normal((n, H, F)).astype(np.float32) for _ in range(4)]
    if dtype == "bf16":
        Q, K, V, g = (synth.bf16_round(x) for x in (Q, K, V, g))
    lay = M.mega_preprocess(ip, ix, num_parts=parts, seg_edges=seg)
    got = _run(lay, Q, K, V, g, dtype)
    f = ogt.gt_forward(ip, ix, Q, K, V)
    ref = {**f, **ogt.gt_backward(ip, ix, Q, K, V, g, fwd=f)}
    for key in ("out", "lse", "grad_q", "grad_k", "grad_v"):
        if dtype == "fp32":
            hz.assert_fp32_close(got[key], ref[key], key)
        else:
            hz.assert_bf16_close(got[key], ref[key], key)


@pytest.mark.parametrize("H,F", [(8, 16), (4, 32), (4, 64), (4, 128), (1, 256), (2, 32)])
def test_gt_bf16_random_multigraph(cuda_device, H, F):
    """bf16 path, split rows and sources (S = 16) and every group width (G = 8, 16, 32; V = 1, 2)."""
    ip, ix = synth.random_multigraph(21, 900, 12000, undirected=False, isolated=15)
    _check(ip, ix, H, F, seed=H * 1000 + F + 7, dtype="bf16", seg=16)


def test_gt_bf16_paper_batch_and_multipart(cuda_device):
    cfg = synth.get_config("zinc-b128")
    ip, ix, _ = synth.make_graph(cfg)
    _check(ip, ix, 8, 16, seed=3, dtype="bf16")
    ip, ix = synth.random_multigraph(4, 500, 6000, undirected=True, isolated=30)
    _check(ip, ix, 4, 32, seed=1, parts=3, dtype="bf16", seg=32)


@pytest.mark.parametrize("H,F", [(8, 16), (4, 32), (1, 8), (2, 100), (4, 128)])
def test_gt_random_multigraph(cuda_device, H, F):
    ip, ix = synth.random_multigraph(21, 900, 12000, undirected=False, isolated=15)
    _check(ip, ix, H, F, seed=H * 1000 + F)


@pytest.mark.parametrize("cfg_name", ["zinc-b128", "csl-b128", "aqsol-b128-drop20"])
def test_gt_paper_batches(cuda_device, cfg_name):
    cfg = synth.get_config(cfg_name)
    ip, ix, _ = synth.make_graph(cfg)
    _check(ip, ix, 8, 16, seed=cfg.seed & 0xFFFF)


def test_gt_multipart_and_edge_cases(cuda_device):
    ip, ix = synth.random_multigraph(4, 500, 6000, undirected=True, isolated=30)
    _check(ip, ix, 4, 16, seed=1, parts=3)
    empty_ip = np.zeros(6, np.int64)
    _check(empty_ip, np.zeros(0, np.int32), 2, 8, seed=2)
