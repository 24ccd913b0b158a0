"""Destination-partitioned multi-GPU GAT layers.

The exact counterpart of the paper's "partition of the path representation
... only two communications for adjacent path partitions":
rank p owns the contiguous, edge-balanced rows [b_p, b_{p+1}) of the MEGA
order (R23) and part p of the layout (its in-edges, every source).

Per layer and step (torch.distributed over NCCL is the plumbing; every
computation is a libmega.so call):
  forward   mega_project_fwd on the owned rows -> all-gather-v of the projected
            rows [Wh | er] (grouped send/recv: partitions are unequal and NCCL
            has no all-gather-v) -> mega_gat_fwd on part p;
  backward  mega_gat_bwd(PHASE_SRC) -> partial dWh and der for every source ->
            reduce of each owner's row block onto its owner -> mega_gat_bwd
            (PHASE_DST) on the owned rows -> mega_project_bwd on the owned rows
            -> all-reduce of dW, da_l, da_r.
The exchange helpers are also exercised on CPU with gloo (tests/test_dist_cpu.py).
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

from . import mega as M
from .layer import GATLayer


def _world(group=None):
    return dist.get_world_size(group) if dist.is_available() and dist.is_initialized() else 1


def allgather_rows(t: torch.Tensor, bounds, group=None):
    """All-gather-v along dim 0: rank q's rows t[b_q:b_{q+1}] are sent to every
    rank, in place (each rank already holds its own block)."""
    if _world(group) == 1:
        return
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    b = [int(x) for x in bounds]
    ops = []
    mine = t[b[rank]:b[rank + 1]]
    for q in range(world):
        if q == rank:
            continue
        peer = dist.get_global_rank(group, q) if group is not None else q   # P2P ops take global ranks
        if b[rank + 1] > b[rank]:
            ops.append(dist.P2POp(dist.isend, mine, peer, group))
        if b[q + 1] > b[q]:
            ops.append(dist.P2POp(dist.irecv, t[b[q]:b[q + 1]], peer, group))
    if ops:
        for r in dist.batch_isend_irecv(ops):
            r.wait()


def reduce_to_owners(t: torch.Tensor, bounds, group=None):
    """Sum t over ranks, block b_q:b_{q+1} landing on its owner q (a reduce-
    scatter-v); other ranks' copies of that block are left unspecified."""
    if _world(group) == 1:
        return
    world = dist.get_world_size(group)
    b = [int(x) for x in bounds]
    for q in range(world):
        if b[q + 1] > b[q]:
            dist.reduce(t[b[q]:b[q + 1]], dst=dist.get_global_rank(group, q) if group else q,
                        op=dist.ReduceOp.SUM, group=group)


class DistGATLayer:
    """One GAT layer on part `rank` of a k-part layout."""

    def __init__(self, layout: M.Layout, rank, x_local, w, attn_l, attn_r, heads, head_dim, in_dim=None,
                 want_grad_x=False, group=None, lp_only=False):
        self.group = group
        self.bounds = layout.view(rank)["bounds"]
        self.L = GATLayer(layout, x_local, w, attn_l, attn_r, heads, head_dim, part=rank, in_dim=in_dim,
                          want_grad_x=want_grad_x, lp_only=lp_only)

    def forward(self, timed=None):
        """timed(name, fn): optional wrapper used by bench.py to time each call."""
        L = self.L
        t = timed or (lambda name, fn: fn())
        t("project_fwd", L.project)
        t("comm_fwd", lambda: (allgather_rows(L.feat, self.bounds, self.group),
                               allgather_rows(L.ctx[1], self.bounds, self.group)))  # [Wh | er] rows
        t("gat_fwd", lambda: L.attend(True))
        return L.out

    def backward(self, grad_out_local, timed=None):
        L = self.L
        t = timed or (lambda name, fn: fn())
        if _world(self.group) == 1:  # one call: lets LP_ONLY keep the partial in the bf16 operand
            t("gat_bwd", lambda: L.attend_backward(grad_out_local, 0))
        else:
            t("gat_bwd_src", lambda: L.attend_backward(grad_out_local, M.MEGA_BWD_PHASE_SRC))
            t("comm_bwd", lambda: (reduce_to_owners(L.grad_feat, self.bounds, self.group),
                                   reduce_to_owners(L.ctx[4], self.bounds, self.group)))  # [dWh | der]
            t("gat_bwd_dst", lambda: L.attend_backward(grad_out_local, M.MEGA_BWD_PHASE_DST))
        t("project_bwd", L.project_backward)
        if _world(self.group) > 1:
            for x in (L.grad_w, L.grad_attn_l, L.grad_attn_r):
                dist.all_reduce(x, group=self.group)
        return L.grad_x
