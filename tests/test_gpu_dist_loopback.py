"""GPU parity of the k-GPU path on one GPU (SURVEY §8(e) "MEGA_LOOPBACK", §4.5).

k ranks are driven by this one process through the library's LOCAL transport
(mega_comm_init_local): every rank keeps its own buffers, as it would on its
own GPU, and the exchange moves the bytes with device-to-device copies instead
of NCCL.  Everything else is the production k-GPU code path of
mega_gat_fwd_dist / mega_gat_bwd_dist: the local/remote split of every row's
in-edges by source owner, block (p,p) computed before the exchange lands, the
remote pass, the fixed-order merge, the source pass for peer-owned sources,
the transfer of their partial [dWh | der] to the owners, the combine and the
destination pass.  Compared element by element with the fp64 oracle on the
whole graph (old ids); the exchanged rows must equal the owners' rows exactly.
"""
import numpy as np
import pytest
import torch

import synth
from oracle import coracle
from paper_conf_icdcs_dengr24_b200 import mega as M
from tests import gpu_harness as hz

pytestmark = pytest.mark.gpu


def run_dist(layout, Wh_old, a_l, a_r, g_old, dtype, dev="cuda"):
    n, H, F = Wh_old.shape
    D = H * F
    v0 = layout.view(0)
    perm = v0["perm"].astype(np.int64)
    k = v0["num_parts"]
    bounds = v0["bounds"]
    tdt = hz.DT[dtype]
    Wh_new = torch.tensor(Wh_old.reshape(n, D)[perm], dtype=torch.float32, device=dev).to(tdt)
    g_new = torch.tensor(g_old.reshape(n, D)[perm], dtype=torch.float32, device=dev).to(tdt)
    al = torch.tensor(a_l.reshape(-1), device=dev)
    ar = torch.tensor(a_r.reshape(-1), device=dev)
    comms = M.mega_comm_init_local(k)
    assert comms[1].info() == {"nranks": k, "rank": 1, "device": torch.cuda.current_device(), "transport": "local"}
    R = []
    for p in range(k):
        layout.bind(p)
        b0, b1 = int(bounds[p]), int(bounds[p + 1])
        feat = torch.zeros(n, D, dtype=tdt, device=dev)       # this rank's global feature array
        feat[b0:b1] = Wh_new[b0:b1]                           # only its own projected rows
        fws, bws = M.mega_gat_dist_workspace_bytes(layout, p, H, F, M._dtype_code(feat))
        R.append({"b0": b0, "b1": b1, "feat": feat, "ctx": torch.zeros(M.MEGA_CTX_PLANES, n, H, device=dev),
                  "out": torch.empty(b1 - b0, D, dtype=tdt, device=dev),
                  "wsf": torch.empty(max(fws, 256), dtype=torch.uint8, device=dev),
                  "wsb": torch.empty(max(bws, 256), dtype=torch.uint8, device=dev),
                  "gf": torch.full((n, D), float("nan"), device=dev), "gal": torch.zeros(D, device=dev),
                  "gar": torch.zeros(D, device=dev), "cs": torch.cuda.Stream()})
    for phase in (M.MEGA_DIST_PHASE_SEND, M.MEGA_DIST_PHASE_RECV):
        for p, r in enumerate(R):   # el/er of the own rows are computed by the call (no ELER_IN_CTX)
            M.mega_gat_fwd_dist(layout, p, comms[p], r["feat"], al, ar, H, F, r["out"], r["ctx"], r["wsf"],
                                flags=phase, comm_stream=r["cs"])
    torch.cuda.synchronize()
    er_owned = torch.cat([r["ctx"][1][r["b0"]:r["b1"]] for r in R])   # er of every row, from its owner
    for p, r in enumerate(R):   # every rank now holds, bit for bit, every row its edges reference (NEXT-1 halo)
        need = torch.tensor(np.unique(layout.view(p)["src"]).astype(np.int64), device=dev)
        assert torch.equal(r["feat"][need], Wh_new[need])
        assert torch.equal(r["ctx"][1][need], er_owned[need])
    for phase in (M.MEGA_DIST_PHASE_SEND, M.MEGA_DIST_PHASE_RECV):
        for p, r in enumerate(R):
            M.mega_gat_bwd_dist(layout, p, comms[p], r["feat"], al, ar, H, F, r["out"], g_new[r["b0"]:r["b1"]],
                                r["ctx"], r["gf"], r["gal"], r["gar"], r["wsb"], flags=phase, comm_stream=r["cs"])
    torch.cuda.synchronize()
    inv = np.empty(n, np.int64)
    inv[perm] = np.arange(n)
    out = torch.cat([r["out"] for r in R]).float().cpu().numpy()
    lse = torch.cat([r["ctx"][2][r["b0"]:r["b1"]] for r in R]).cpu().numpy()
    gf = torch.cat([r["gf"][r["b0"]:r["b1"]] for r in R]).cpu().numpy()
    gal = sum(r["gal"] for r in R).cpu().numpy()    # the caller's all-reduce of the parameter partials
    gar = sum(r["gar"] for r in R).cpu().numpy()
    return {"out": out[inv].reshape(n, H, F), "lse": lse[inv], "grad_feat": gf[inv].reshape(n, H, F),
            "grad_attn_l": gal.reshape(H, F), "grad_attn_r": gar.reshape(H, F)}


@pytest.mark.parametrize("k", [2, 3, 4])
@pytest.mark.parametrize("dtype", ["fp32", "bf16"])
def test_dist_loopback_reddit_shaped(cuda_device, dtype, k):
    cfg = synth.scaled(synth.CONFIGS["reddit"], 3000, 120000)
    ip, ix, _ = synth.make_graph(cfg)
    Wh, a_l, a_r, g = hz.inputs(9, cfg.n, 4, 64, dtype == "bf16")
    lay = M.mega_preprocess(ip, ix, num_parts=k, seg_edges=200)   # hubs split across segments and passes
    dv = [M.mega_layout_dist_view_get(lay, p) for p in range(k)]
    assert all(d["num_local_items"] > 0 and d["num_remote_items"] > 0 for d in dv)
    assert any(d["num_splits"] > 0 for d in dv)
    got = run_dist(lay, Wh, a_l, a_r, g, dtype)
    f = coracle.gat_forward(ip, ix, Wh, a_l, a_r)
    ref = {**f, **coracle.gat_backward(ip, ix, Wh, a_l, a_r, g, fwd=f)}
    hz.check(got, ref, dtype, graph=(ip, ix, Wh, a_l, a_r, g))


@pytest.mark.parametrize("dtype", ["fp32", "bf16"])
def test_dist_loopback_random_multigraph(cuda_device, dtype):
    ip, ix = synth.random_multigraph(17, 900, 12000, undirected=False, isolated=30)
    n = len(ip) - 1
    Wh, a_l, a_r, g = hz.inputs(4, n, 4, 32, dtype == "bf16")
    lay = M.mega_preprocess(ip, ix, num_parts=3, seg_edges=16)
    got = run_dist(lay, Wh, a_l, a_r, g, dtype)
    f = coracle.gat_forward(ip, ix, Wh, a_l, a_r)
    ref = {**f, **coracle.gat_backward(ip, ix, Wh, a_l, a_r, g, fwd=f)}
    hz.check(got, ref, dtype, graph=(ip, ix, Wh, a_l, a_r, g))
    deg = np.diff(ip)
    assert np.all(got["out"][deg == 0] == 0) and np.all(got["lse"][deg == 0] == -np.inf)


def test_nccl_comm_single_rank(cuda_device):
    """The NCCL transport loads libnccl (dlopen), bootstraps from a unique id and runs the
    dist entry points (k = 1: no messages) -- the multi-rank NCCL path needs several GPUs."""
    uid = M.mega_comm_unique_id()
    assert len(uid) == 128
    comm = M.mega_comm_init(uid, 1, 0, torch.cuda.current_device())
    assert comm.info()["transport"] == "nccl" and comm.info()["nranks"] == 1
    ip, ix = synth.random_multigraph(3, 300, 3000)
    n = len(ip) - 1
    Wh, a_l, a_r, g = hz.inputs(2, n, 4, 32, False)
    lay = M.mega_preprocess(ip, ix)
    lay.bind(0)
    perm = lay.view(0)["perm"].astype(np.int64)
    feat = torch.tensor(Wh.reshape(n, -1)[perm], device="cuda")
    ctx = torch.zeros(M.MEGA_CTX_PLANES, n, 4, device="cuda")
    out = torch.empty(n, 128, device="cuda")
    fws, _ = M.mega_gat_dist_workspace_bytes(lay, 0, 4, 32, M.MEGA_F32)
    ws = torch.empty(max(fws, 256), dtype=torch.uint8, device="cuda")
    M.mega_gat_fwd_dist(lay, 0, comm, feat, torch.tensor(a_l.reshape(-1), device="cuda"),
                        torch.tensor(a_r.reshape(-1), device="cuda"), 4, 32, out, ctx, ws, comm_stream=torch.cuda.Stream())
    torch.cuda.synchronize()
    inv = np.empty(n, np.int64)
    inv[perm] = np.arange(n)
    ref = coracle.gat_forward(ip, ix, Wh, a_l, a_r)
    hz.assert_fp32_close(out.cpu().numpy()[inv], ref["out"].reshape(n, -1), "out")


@pytest.mark.parametrize("k", [2, 3])
def test_dist_whole_layer_bf16(cuda_device, k):
    """dist.DistGATLayer (what bench.py runs on k GPUs) end to end on one GPU through the LOCAL
    transport: tcgen05 projection of the own rows, halo exchange + split forward, split backward,
    projection backward; the summed parameter partials stand in for the all-reduce."""
    from oracle import gat as og
    from paper_conf_icdcs_dengr24_b200.dist import DistGATLayer
    cfg = synth.scaled(synth.CONFIGS["products"], 4000, 80000)
    ip, ix, _ = synth.make_graph(cfg)
    inp = synth.make_layer_inputs(cfg)
    x, w, g = synth.bf16_round(inp["x"]), synth.bf16_round(inp["w"]), synth.bf16_round(inp["grad_out"])
    H, F, D, n = cfg.heads, cfg.head_dim, cfg.dim, cfg.n
    lay = M.mega_preprocess(ip, ix, num_parts=k)
    perm = lay.view(0)["perm"].astype(np.int64)
    bounds = lay.view(0)["bounds"]
    comms = M.mega_comm_init_local(k)
    layers = []
    for p in range(k):
        lay.bind(p)
        b0, b1 = int(bounds[p]), int(bounds[p + 1])
        xt = torch.tensor(x[perm][b0:b1], device="cuda").bfloat16().contiguous()
        layers.append(DistGATLayer(lay, p, xt, torch.tensor(w, device="cuda").bfloat16(),
                                   torch.tensor(inp["a_l"], device="cuda"), torch.tensor(inp["a_r"], device="cuda"),
                                   H, F, in_dim=inp["in_dim"], want_grad_x=True, lp_only=True, comm=comms[p]))
    gn = torch.tensor(g[perm], device="cuda").bfloat16()
    for phase in (M.MEGA_DIST_PHASE_SEND, M.MEGA_DIST_PHASE_RECV):
        for Ld in layers:
            Ld.forward(phase=phase)
    for phase in (M.MEGA_DIST_PHASE_SEND, M.MEGA_DIST_PHASE_RECV):
        for p, Ld in enumerate(layers):
            Ld.backward(gn[int(bounds[p]):int(bounds[p + 1])], phase=phase)
    torch.cuda.synchronize()
    inv = np.empty(n, np.int64)
    inv[perm] = np.arange(n)
    Wh = synth.bf16_round(og.project_forward(x, w).astype(np.float32)).astype(np.float64).reshape(n, H, F)
    f = coracle.gat_forward(ip, ix, Wh, inp["a_l"], inp["a_r"])
    b = coracle.gat_backward(ip, ix, Wh, inp["a_l"], inp["a_r"], g.reshape(n, H, F), fwd=f)
    pb = og.project_backward(x, w, b["grad_feat"].reshape(n, D))
    out = torch.cat([Ld.L.out for Ld in layers]).float().cpu().numpy()[inv]
    gx = torch.cat([Ld.L.grad_x for Ld in layers]).float().cpu().numpy()[inv]
    hz.assert_bf16_close(out, f["out"].reshape(n, D), "out")
    hz.assert_bf16_close(gx, pb["grad_x"], "grad_x")
    for name, ref in (("grad_w", pb["grad_w"]), ("grad_attn_l", b["grad_attn_l"].reshape(-1)),
                      ("grad_attn_r", b["grad_attn_r"].reshape(-1))):
        got = sum(getattr(Ld.L, name) for Ld in layers).cpu().numpy()
        hz.assert_bf16_close(got, ref, name)
