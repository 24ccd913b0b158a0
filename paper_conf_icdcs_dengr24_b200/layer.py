"""One GAT layer (a2-a9) on one part, driving libmega.so through the binding.

torch supplies the device buffers and the stream; every computation is a
libmega.so call (mega_project_fwd -> mega_gat_fwd -> mega_gat_bwd ->
mega_project_bwd).  Features live in the layout's new (traversal) order.
"""
from __future__ import annotations

import torch

from . import mega as M


class GATLayer:
    """Buffers and calls for one layer on one layout part (k = 1: the whole graph)."""

    def __init__(self, layout: M.Layout, x, w, attn_l, attn_r, heads, head_dim, part=0, in_dim=None,
                 negative_slope=M.SLOPE, want_grad_x=False, lp_only=False):
        self.layout, self.part = layout, part
        self.lp_only = lp_only  # training path: only the bf16 operand of the projection backward is needed
        view_counts = layout.view(part, arrays=False)
        self.n = view_counts["num_nodes"]
        self.row_begin, self.row_end = view_counts["row_begin"], view_counts["row_end"]
        self.rows = self.row_end - self.row_begin
        self.x, self.w = x, w
        self.in_dim = in_dim or w.shape[0]
        self.attn_l = attn_l.reshape(-1).float().contiguous()
        self.attn_r = attn_r.reshape(-1).float().contiguous()
        self.H, self.F = heads, head_dim
        self.D = heads * head_dim
        self.slope = negative_slope
        self.dtype = x.dtype
        dev = x.device
        D, n = self.D, self.n
        self.feat = torch.empty(n, D, dtype=self.dtype, device=dev)
        self.ctx = torch.zeros(M.MEGA_CTX_PLANES, n, heads, dtype=torch.float32, device=dev)
        self.out = torch.empty(self.rows, D, dtype=self.dtype, device=dev)
        fws, bws = M.mega_gat_workspace_bytes(layout, part, heads, head_dim, M._dtype_code(x))
        self.ws_f = torch.empty(max(fws, 256), dtype=torch.uint8, device=dev)
        self.ws_b = torch.empty(max(bws, 256), dtype=torch.uint8, device=dev)
        self.grad_feat = torch.empty(n, D, dtype=torch.float32, device=dev)
        self.grad_feat_lp = torch.empty(n, D, dtype=self.dtype, device=dev) if self.dtype == torch.bfloat16 else None
        self.grad_attn_l = torch.empty(D, dtype=torch.float32, device=dev)
        self.grad_attn_r = torch.empty(D, dtype=torch.float32, device=dev)
        # rows >= in_dim (zero padding of W) are never written by mega_project_bwd: keep them 0
        self.grad_w = torch.zeros(self.w.shape[0], D, dtype=torch.float32, device=dev)
        self.grad_x = torch.empty_like(self.x) if want_grad_x else None
        pws = M.mega_project_workspace_bytes(self.x.shape[0], self.in_dim, heads, head_dim, M._dtype_code(x))
        self.ws_p = torch.empty(max(pws, 256), dtype=torch.uint8, device=dev)

    # a2
    def project(self, stream=None):
        M.mega_project_fwd(self.x, self.w, self.attn_l, self.attn_r, self.H, self.F,
                           self.feat[self.row_begin:self.row_end] if self.x.shape[0] != self.n else self.feat,
                           self.ctx, self.n, self.row_begin if self.x.shape[0] != self.n else 0,
                           in_dim=self.in_dim, stream=stream)

    # a3-a5
    def attend(self, eler_in_ctx=True, stream=None):
        M.mega_gat_fwd(self.layout, self.part, self.feat, self.attn_l, self.attn_r, self.H, self.F, self.out,
                       self.ctx, self.ws_f, self.slope, M.MEGA_FLAG_ELER_IN_CTX if eler_in_ctx else 0, stream)

    # a6-a8
    def attend_backward(self, grad_out, flags=0, stream=None):
        if self.lp_only and self.grad_feat_lp is not None:
            flags |= M.MEGA_BWD_LP_ONLY
        M.mega_gat_bwd(self.layout, self.part, self.feat, self.attn_l, self.attn_r, self.H, self.F, self.out,
                       grad_out, self.ctx, self.grad_feat, self.grad_attn_l, self.grad_attn_r, self.ws_b,
                       self.grad_feat_lp, self.slope, flags, stream)

    # a9
    def project_backward(self, stream=None):
        gf = self.grad_feat_lp if self.dtype == torch.bfloat16 else self.grad_feat
        rows = slice(self.row_begin, self.row_end) if self.x.shape[0] != self.n else slice(None)
        M.mega_project_bwd(self.x, self.w, self.H, self.F, gf[rows], self.grad_w, self.grad_x,
                           in_dim=self.in_dim, ws=self.ws_p, stream=stream)

    def forward(self, stream=None):
        self.project(stream)
        self.attend(True, stream)
        return self.out

    def backward(self, grad_out, stream=None):
        self.attend_backward(grad_out, 0, stream)
        self.project_backward(stream)

    def step(self, grad_out, stream=None):
        self.forward(stream)
        self.backward(grad_out, stream)

    def launches_per_step(self) -> int:
        """Our kernels per step.  bf16: projection GEMM (el/er in its epilogue), fwd, [fwd merge], dlt,
        bwd_src, [bwd_src merge], bwd_dst, reduce(a_l, a_r), dW GEMM + its reduce, [dX GEMM].
        fp32: eler, fwd, [merge], dlt, bwd_src, [merge], bwd_dst, reduce (the fp32 GEMMs are cuBLAS's)."""
        v = self.layout.view(self.part, arrays=False)
        splits = (1 if v["num_fwd_splits"] > 0 else 0) + (1 if v["num_bwd_splits"] > 0 else 0)
        if self.dtype == torch.bfloat16:
            return 8 + splits + (1 if self.grad_x is not None else 0)
        return 6 + splits
