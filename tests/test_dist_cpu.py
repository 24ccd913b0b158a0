"""Multi-GPU host logic on CPU: world-size-2 gloo process group.

The k-GPU path (paper_conf_icdcs_dengr24_b200/dist.py) splits one GAT layer by
destination partitions of the MEGA order (R23): each
rank computes its rows' forward from all-gathered source rows, a partial
backward over its own edges for every source, sums the partials onto their
owners, and all-reduces the parameter gradients.  Here the product's layout
parts (mega_preprocess, host code) and the product's exchange helpers
(allgather_rows, reduce_to_owners over gloo) carry the oracle's per-part fp64
arithmetic, and the assembled result must equal the single-process oracle.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth
from oracle import gat as og
from paper_conf_icdcs_dengr24_b200 import dist as D
from paper_conf_icdcs_dengr24_b200 import mega as M


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        ip, ix = synth.random_multigraph(21, 300, 3000, undirected=True, isolated=5)
        n = len(ip) - 1
        H, F = 2, 4
        rng = np.random.default_rng(3)
        Wh_old = rng.standard_normal((n, H, F))
        a_l = rng.standard_normal((H, F))
        a_r = rng.standard_normal((H, F))
        g_old = rng.standard_normal((n, H, F))
        lay = M.mega_preprocess(ip, ix, num_parts=world, seg_edges=16)
        v = lay.view(rank)
        perm = v["perm"].astype(np.int64)
        b = v["bounds"]
        b0, b1 = int(v["row_begin"]), int(v["row_end"])
        Wh = Wh_old[perm]
        g = g_old[perm]
        # part-p subgraph in new ids: rows outside the part have no in-edges
        ip_p = np.zeros(n + 1, np.int64)
        ip_p[b0 + 1:b1 + 1] = v["indptr"][1:]
        ip_p[b1 + 1:] = v["indptr"][-1]
        src_p = v["src"]
        # forward: every rank "projects" its own rows, then all-gathers them
        feat = torch.zeros(n, H * F, dtype=torch.float64)
        feat[b0:b1] = torch.from_numpy(Wh[b0:b1].reshape(-1, H * F))
        D.allgather_rows(feat, b)
        assert torch.equal(feat, torch.from_numpy(Wh.reshape(n, H * F)))
        fwd = og.gat_forward(ip_p, src_p, feat.numpy().reshape(n, H, F), a_l, a_r)
        # backward: partial over this part's edges for every source, summed onto owners
        bwd = og.gat_backward(ip_p, src_p, Wh, a_l, a_r, g, fwd=fwd)
        gf = torch.from_numpy(np.ascontiguousarray(bwd["grad_feat"].reshape(n, H * F)))
        D.reduce_to_owners(gf, b)
        gal = torch.from_numpy(np.ascontiguousarray(bwd["grad_attn_l"]))
        gar = torch.from_numpy(np.ascontiguousarray(bwd["grad_attn_r"]))
        dist.all_reduce(gal)
        dist.all_reduce(gar)
        # reference: single-process oracle on the whole graph (new ids)
        ip_all, src_all = _relabel_ptr(lay), _all_src(lay)
        ref_f = og.gat_forward(ip_all, src_all, Wh, a_l, a_r)
        ref_b = og.gat_backward(ip_all, src_all, Wh, a_l, a_r, g, fwd=ref_f)
        ok_out = np.allclose(fwd["out"][b0:b1], ref_f["out"][b0:b1], rtol=1e-12, atol=1e-12)
        ok_gf = np.allclose(gf.numpy()[b0:b1], ref_b["grad_feat"].reshape(n, -1)[b0:b1], rtol=1e-11, atol=1e-11)
        ok_al = np.allclose(gal.numpy(), ref_b["grad_attn_l"], rtol=1e-11, atol=1e-11)
        ok_ar = np.allclose(gar.numpy(), ref_b["grad_attn_r"], rtol=1e-11, atol=1e-11)
        q.put((rank, ok_out, ok_gf, ok_al, ok_ar, b1 - b0, len(src_p)))
    finally:
        dist.destroy_process_group()


def _relabel_ptr(lay):
    parts = [lay.view(p) for p in range(lay.view(0)["num_parts"])]
    n = parts[0]["num_nodes"]
    ip = np.zeros(n + 1, np.int64)
    off = 0
    for v in parts:
        b0, b1 = int(v["row_begin"]), int(v["row_end"])
        ip[b0 + 1:b1 + 1] = v["indptr"][1:] + off
        off += int(v["indptr"][-1])
    return ip


def _all_src(lay):
    parts = [lay.view(p) for p in range(lay.view(0)["num_parts"])]
    return np.concatenate([v["src"] for v in parts])


@pytest.mark.parametrize("world", [2])
def test_partitioned_layer_equals_single_process(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(p.exitcode == 0 for p in procs)
    for rank, ok_out, ok_gf, ok_al, ok_ar, rows, edges in res:
        assert ok_out and ok_gf and ok_al and ok_ar, (rank, ok_out, ok_gf, ok_al, ok_ar)
        assert rows > 0 and edges > 0


def _subgroup_worker(rank, world, port, q):
    """allgather_rows on a subgroup whose group ranks differ from the global ranks."""
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        sub = dist.new_group([1, 2])
        if rank in (1, 2):
            gr = dist.get_rank(sub)            # 0 or 1
            bounds = [0, 3, 7]
            t = torch.zeros(7, 2)
            t[bounds[gr]:bounds[gr + 1]] = float(rank)
            D.allgather_rows(t, bounds, group=sub)
            ok = torch.equal(t[:3], torch.full((3, 2), 1.0)) and torch.equal(t[3:], torch.full((4, 2), 2.0))
            q.put((rank, ok))
        dist.barrier()
    finally:
        dist.destroy_process_group()


def test_allgather_rows_on_a_subgroup():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_subgroup_worker, args=(r, 3, port, q)) for r in range(3)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
    assert all(p.exitcode == 0 for p in procs)
    assert all(ok for _, ok in res), res
