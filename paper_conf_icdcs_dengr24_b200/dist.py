"""Destination-partitioned multi-GPU GAT layers.

The exact counterpart of the paper's "partition of the path representation
... only two communications for adjacent path partitions":
rank p owns the contiguous, edge-balanced rows [b_p, b_{p+1}) of the MEGA
order (R23) and part p of the layout (its in-edges, every source).

Per layer and step, every computation and every byte of the exchange is a
libmega.so call on a library-owned communicator (include/mega.h "k GPUs"):
  forward   mega_project_fwd on the owned rows -> mega_gat_fwd_dist: the
            [Wh | er] rows travel to every peer on a comm stream while block
            (p,p) is aggregated, then the remote blocks and the merge;
  backward  mega_gat_bwd_dist: partial [dWh | der] of the peers' sources travel
            to their owners while this rank's own sources are processed, then
            the destination pass -> mega_project_bwd on the owned rows.
torch.distributed is the plumbing only: it broadcasts the 128-byte NCCL id
that bootstraps the library's communicator, and all-reduces the parameter
gradients (dW, da_l, da_r) as data-parallel training does.

allgather_rows / reduce_to_owners are the same exchange written with
torch.distributed point-to-point ops; the CPU (gloo) test uses them to check
the partition semantics against the oracle without a GPU.
"""
from __future__ import annotations

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


def make_comm(group=None) -> M.Comm:
    """Bootstrap the library-owned NCCL communicator from the torch process group:
    rank 0 draws the unique id, torch broadcasts it, every rank joins."""
    world, rank = dist.get_world_size(group), dist.get_rank(group)
    obj = [M.mega_comm_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
    return M.mega_comm_init(obj[0], world, rank, torch.cuda.current_device())


class DistGATLayer:
    """One GAT layer on part `rank` of a k-part layout (k = 1: the single-GPU layer)."""

    def __init__(self, layout: M.Layout, rank, x_local, w, attn_l, attn_r, heads, head_dim, in_dim=None,
                 want_grad_x=False, group=None, lp_only=False, comm: M.Comm | None = None):
        self.group = group
        self.rank = rank
        self.k = layout.view(rank, arrays=False)["num_parts"]
        self.comm = comm
        if self.k > 1 and comm is None:
            raise ValueError("a k-part layout needs a mega communicator (dist.make_comm)")
        self.L = GATLayer(layout, x_local, w, attn_l, attn_r, heads, head_dim, part=rank, in_dim=in_dim,
                          want_grad_x=want_grad_x, lp_only=lp_only)
        if self.k > 1:
            L = self.L
            fws, bws = M.mega_gat_dist_workspace_bytes(layout, rank, heads, head_dim, M._dtype_code(x_local))
            L.ws_f = torch.empty(max(fws, 256), dtype=torch.uint8, device=x_local.device)
            L.ws_b = torch.empty(max(bws, 256), dtype=torch.uint8, device=x_local.device)
            self.cs = torch.cuda.Stream(device=x_local.device)
        # parameter gradients all-reduced in one flat buffer
        L = self.L
        self._pg = [L.grad_w, L.grad_attn_l, L.grad_attn_r]

    def forward(self, timed=None, phase=0):
        """timed(name, fn): optional wrapper used by bench.py to time each call.
        phase: 0 (both halves), or MEGA_DIST_PHASE_SEND / _RECV for a driver that runs every
        rank in one process (the LOCAL transport): SEND projects and posts, RECV finishes."""
        L = self.L
        t = timed or (lambda name, fn: fn())
        if phase != M.MEGA_DIST_PHASE_RECV:
            t("project_fwd", L.project)
        if self.k == 1:
            t("gat_fwd", lambda: L.attend(True))
        else:   # exchange of [Wh | er] overlapped with block (p, p), remote blocks, merge
            t("gat_fwd", lambda: M.mega_gat_fwd_dist(L.layout, self.rank, self.comm, L.feat, L.attn_l, L.attn_r, L.H,
                                                     L.F, L.out, L.ctx, L.ws_f, L.slope,
                                                     M.MEGA_FLAG_ELER_IN_CTX | phase, comm_stream=self.cs))
        return L.out

    def backward(self, grad_out_local, timed=None, split=False, phase=0):
        """split (k = 1): the source and destination phases as two calls, for per-phase timing
        (the same work as the single call).  phase: as in forward (k > 1; the RECV half runs the
        projection backward and the parameter all-reduce)."""
        L = self.L
        t = timed or (lambda name, fn: fn())
        if self.k > 1 and phase:
            flags = M.MEGA_BWD_LP_ONLY if (L.lp_only and L.grad_feat_lp is not None) else 0
            t("gat_bwd", lambda: M.mega_gat_bwd_dist(L.layout, self.rank, self.comm, L.feat, L.attn_l, L.attn_r, L.H,
                                                     L.F, L.out, grad_out_local, L.ctx, L.grad_feat, L.grad_attn_l,
                                                     L.grad_attn_r, L.ws_b, L.grad_feat_lp, L.slope, flags | phase,
                                                     comm_stream=self.cs))
            if phase == M.MEGA_DIST_PHASE_SEND:
                return None
            t("project_bwd", L.project_backward)
            if _world(self.group) > 1:
                t("allreduce_params", self._allreduce_params)
            return L.grad_x
        if self.k == 1 and split:
            t("gat_bwd_src", lambda: L.attend_backward(grad_out_local, M.MEGA_BWD_PHASE_SRC))
            t("gat_bwd_dst", lambda: L.attend_backward(grad_out_local, M.MEGA_BWD_PHASE_DST))
        elif self.k == 1:   # one call: lets LP_ONLY keep the partial in the bf16 operand
            t("gat_bwd", lambda: L.attend_backward(grad_out_local, 0))
        else:
            flags = M.MEGA_BWD_LP_ONLY if (L.lp_only and L.grad_feat_lp is not None) else 0
            t("gat_bwd", lambda: M.mega_gat_bwd_dist(L.layout, self.rank, self.comm, L.feat, L.attn_l, L.attn_r, L.H,
                                                     L.F, L.out, grad_out_local, L.ctx, L.grad_feat, L.grad_attn_l,
                                                     L.grad_attn_r, L.ws_b, L.grad_feat_lp, L.slope, flags,
                                                     comm_stream=self.cs))
        t("project_bwd", L.project_backward)
        if _world(self.group) > 1:
            t("allreduce_params", self._allreduce_params)
        return L.grad_x

    def _allreduce_params(self):
        flat = torch.cat([p.reshape(-1) for p in self._pg])
        dist.all_reduce(flat, group=self.group)
        off = 0
        for p in self._pg:
            p.copy_(flat[off:off + p.numel()].view_as(p))
            off += p.numel()
