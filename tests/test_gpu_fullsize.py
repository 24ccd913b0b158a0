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


def _wh(x, w, nodes, H, F):
    return synth.bf16_round((x[nodes].astype(np.float64) @ w.astype(np.float64)).astype(np.float32)).reshape(
        len(nodes), H, F)


@pytest.mark.parametrize("name", ["products", "reddit"])
def test_fullsize_sampled(cuda_device, name):
    cfg = synth.CONFIGS[name]
    ip, ix, _ = synth.make_graph(cfg)
    inp = synth.make_layer_inputs(cfg)
    x, w = synth.bf16_round(inp["x"]), synth.bf16_round(inp["w"])
    g = synth.bf16_round(inp["grad_out"])
    H, F, D, n = cfg.heads, cfg.head_dim, cfg.dim, cfg.n
    import bench
    lay = M.mega_preprocess(ip, ix, block_rows=bench.block_rows_for(cfg, "bf16"))  # bench's layout options
    lay.bind(0)
    perm = lay.view(0)["perm"].astype(np.int64)
    L = hz.layer(lay, x[perm], w, inp["a_l"], inp["a_r"], H, F, "bf16", want_grad_x=False)
    L.step(torch.tensor(g[perm], device="cuda").bfloat16())
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
    f = coracle.gat_forward(ip_c, ix_c, _wh(x, w, nodes, H, F), inp["a_l"], inp["a_r"])
    got_out = L.out[torch.tensor(new_of_old[rows], device="cuda")].float().cpu().numpy()
    got_lse = L.ctx[2][torch.tensor(new_of_old[rows], device="cuda")].cpu().numpy()
    hz.assert_bf16_close(got_out, f["out"][:len(rows)].reshape(len(rows), D), "out")
    fin = np.isfinite(f["lse"][:len(rows)])
    assert np.array_equal(fin, np.isfinite(got_lse)), "lse finiteness"
    hz.assert_bf16_close(got_lse[fin], f["lse"][:len(rows)][fin], "lse")
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
    ref = coracle.gat_backward_srcs(ip_c, ix_c, _wh(x, w, nodes, H, F), inp["a_l"], inp["a_r"], g_c,
                                    [cid[int(s)] for s in srcs])
    got = L.grad_feat[torch.tensor(new_of_old[srcs], device="cuda")].cpu().numpy()
    hz.assert_bf16_close(got, ref.reshape(len(srcs), D), "grad_feat")
