"""Full-size GPU parity at BASELINE.json sizes, in bench.py's launch
configuration (bf16 storage, auto layout options, GATLayer through the C ABI).

The oracle cannot redo a 62M/115M-edge layer element by element in a test, so
it checks sampled outputs it can compute one by one (③):
destination rows (out, lse) and source rows (grad_feat), chosen to include the
largest in-degree / out-degree rows (split into segments and merged), rows
without in-edges, and random rows.  Everything the oracle needs is rebuilt
from the input CSR in OLD node ids and the seeded inputs: Wh = bf16(X W) in
fp64 for the rows involved (DESIGN.md R-prec), never from the GPU.
"""
import numpy as np
import pytest
import torch

import synth
from oracle import coracle
from oracle import gat as og
from paper_conf_icdcs_dengr24_b200 import mega as M
from tests import gpu_harness as hz

pytestmark = pytest.mark.gpu


def _compact(ip, ix, rows):
    """Subgraph holding the in-edges of `rows` (old ids), relabelled compactly.
    Returns (ip_c, ix_c, nodes) with nodes[k] = old id of compact id k and rows
    mapped to compact ids 0..len(rows)-1."""
    rows = np.asarray(rows, np.int64)
    srcs = np.concatenate([ix[ip[r]:ip[r + 1]] for r in rows]) if len(rows) else np.zeros(0, np.int64)
    nodes = np.concatenate([rows, np.setdiff1d(np.unique(srcs), rows)])
    cmap = np.full(len(ip) - 1, -1, np.int64)
    cmap[nodes] = np.arange(len(nodes))
    ip_c = np.zeros(len(nodes) + 1, np.int64)
    ip_c[1:len(rows) + 1] = np.cumsum(ip[rows + 1] - ip[rows])
    ip_c[len(rows) + 1:] = ip_c[len(rows)]
    return ip_c, cmap[srcs].astype(np.int32), nodes


def _wh(x, w, nodes, H, F, dtype="bf16"):
    wh = x[nodes].astype(np.float64) @ w.astype(np.float64)
    # bf16 mode: the GPU stores Wh in bf16 (DESIGN.md R-prec); fp32 mode: true fp32 GEMM, oracle exact
    return (synth.bf16_round(wh.astype(np.float32)) if dtype == "bf16" else wh).reshape(len(nodes), H, F)


def _close(dtype):
    return hz.assert_bf16_close if dtype == "bf16" else hz.assert_fp32_close


@pytest.mark.parametrize("name,dtype", [("products", "bf16"), ("reddit", "bf16"), ("products", "fp32")])
def test_fullsize_sampled(cuda_device, name, dtype):
    cfg = synth.CONFIGS[name]
    ip, ix, _ = synth.make_graph(cfg)
    inp = synth.make_layer_inputs(cfg)
    x, w, g = inp["x"], inp["w"], inp["grad_out"]
    if dtype == "bf16":
        x, w, g = synth.bf16_round(x), synth.bf16_round(w), synth.bf16_round(g)
    H, F, D, n = cfg.heads, cfg.head_dim, cfg.dim, cfg.n
    import bench
    lay = M.mega_preprocess(ip, ix, block_rows=bench.block_rows_for(cfg, dtype))  # bench's layout options
    lay.bind(0)
    perm = lay.view(0)["perm"].astype(np.int64)
    L = hz.layer(lay, x[perm], w, inp["a_l"], inp["a_r"], H, F, dtype, want_grad_x=False)
    L.lp_only = dtype == "bf16"                         # bench's training path
    L.step(torch.tensor(g[perm], device="cuda").to(hz.DT[dtype]).contiguous())
    torch.cuda.synchronize()
    new_of_old = np.empty(n, np.int64)
    new_of_old[perm] = np.arange(n)
    indeg = np.diff(ip)
    outdeg = np.bincount(ix, minlength=n)
    rng = np.random.default_rng(0)
    # ---- forward: sampled destination rows ----
    rows = np.unique(np.concatenate([np.argsort(-indeg)[:4], np.flatnonzero(indeg == 0)[:4],
                                     rng.integers(0, n, 40)]))
    ip_c, ix_c, nodes = _compact(ip, ix, rows)
    f = coracle.gat_forward(ip_c, ix_c, _wh(x, w, nodes, H, F, dtype), inp["a_l"], inp["a_r"])
    got_out = L.out[torch.tensor(new_of_old[rows], device="cuda")].float().cpu().numpy()
    got_lse = L.ctx[2][torch.tensor(new_of_old[rows], device="cuda")].cpu().numpy()
    _close(dtype)(got_out, f["out"][:len(rows)].reshape(len(rows), D), "out")
    fin = np.isfinite(f["lse"][:len(rows)])
    assert np.array_equal(fin, np.isfinite(got_lse)), "lse finiteness"
    _close(dtype)(got_lse[fin], f["lse"][:len(rows)][fin], "lse")
    # ---- backward: sampled source rows (dWh_j needs every out-neighbour's row and j's own row) ----
    hubs = np.argsort(-outdeg)[:2] if name == "products" else np.argsort(-outdeg)[200:201]
    srcs = np.unique(np.concatenate([hubs, rng.integers(0, n, 6)]))
    order = np.argsort(ix, kind="stable")
    cptr = np.zeros(n + 1, np.int64)
    cptr[1:] = np.cumsum(outdeg)
    dst_of_edge = np.repeat(np.arange(n), indeg)[order]
    need = np.unique(np.concatenate([srcs] + [dst_of_edge[cptr[s]:cptr[s + 1]] for s in srcs]))
    ip_c, ix_c, nodes = _compact(ip, ix, need)
    cid = {int(v): k for k, v in enumerate(nodes[:len(need)])}
    g_c = np.zeros((len(nodes), H, F), np.float32)
    g_c[:len(need)] = g[need].reshape(len(need), H, F)
    ref = coracle.gat_backward_srcs(ip_c, ix_c, _wh(x, w, nodes, H, F, dtype), inp["a_l"], inp["a_r"], g_c,
                                    [cid[int(s)] for s in srcs])
    # bf16 training path (LP_ONLY): the final dWh rows are the bf16 GEMM operand grad_feat_lp
    gf = L.grad_feat if dtype == "fp32" else L.grad_feat_lp
    got = gf[torch.tensor(new_of_old[srcs], device="cuda")].float().cpu().numpy()
    _close(dtype)(got, ref.reshape(len(srcs), D), "grad_feat")


def test_fullsize_reddit_parameter_grads(cuda_device):
    """Whole-tensor parity of the parameter gradients at full Reddit size (114.6M
    edges): grad_attn_l, grad_attn_r and grad_w from one bf16 layer fwd+bwd in
    bench's launch configuration, against the full fp64 C oracle (OpenMP) on the
    same seeded inputs, Wh = bf16(X W) computed in fp64 (DESIGN.md R-prec)."""
    cfg = synth.CONFIGS["reddit"]
    ip, ix, _ = synth.make_graph(cfg)
    inp = synth.make_layer_inputs(cfg)
    x, w, g = synth.bf16_round(inp["x"]), synth.bf16_round(inp["w"]), synth.bf16_round(inp["grad_out"])
    H, F, D, n = cfg.heads, cfg.head_dim, cfg.dim, cfg.n
    import bench
    lay = M.mega_preprocess(ip, ix, block_rows=bench.block_rows_for(cfg, "bf16"))
    lay.bind(0)
    perm = lay.view(0)["perm"].astype(np.int64)
    L = hz.layer(lay, x[perm], w, inp["a_l"], inp["a_r"], H, F, "bf16", want_grad_x=False)
    L.lp_only = True                                    # bench's training path
    L.step(torch.tensor(g[perm], device="cuda").bfloat16())
    torch.cuda.synchronize()
    Wh = _wh(x, w, np.arange(n), H, F)
    f = coracle.gat_forward(ip, ix, Wh, inp["a_l"], inp["a_r"])
    b = coracle.gat_backward(ip, ix, Wh, inp["a_l"], inp["a_r"], g.reshape(n, H, F), fwd=f)
    hz.assert_bf16_close(L.grad_attn_l.cpu().numpy(), b["grad_attn_l"].reshape(-1), "grad_attn_l")
    hz.assert_bf16_close(L.grad_attn_r.cpu().numpy(), b["grad_attn_r"].reshape(-1), "grad_attn_r")
    grad_w = x.astype(np.float64).T @ b["grad_feat"].reshape(n, D)
    hz.assert_bf16_close(L.grad_w.cpu().numpy(), grad_w, "grad_w")
