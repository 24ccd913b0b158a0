"""Thin Python binding of libmega.so (include/mega.h) — argument marshalling only.

Every function here has the name of the C entry point it calls.  PyTorch is
used for device memory and streams only; every step of the hot path runs in
libmega.so's kernels.  There is no fallback: if libmega.so is missing or the
device is not an sm_100 GPU the calls raise.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libmega.so")

MEGA_F32, MEGA_BF16 = 0, 1
ORDERS = {"traversal": 0, "identity": 1, "degree": 2, "random": 3}
MEGA_FLAG_ELER_IN_CTX = 1
MEGA_CTX_PLANES = 5  # el, er, lse, Dlt, der
MEGA_BWD_PHASE_SRC = 2
MEGA_BWD_PHASE_DST = 4
MEGA_BWD_LP_ONLY = 8
MEGA_DIST_PHASE_SEND = 16
MEGA_DIST_PHASE_RECV = 32
SLOPE = float(np.float32(0.2))

_c = ctypes
P = _c.c_void_p
I64 = _c.c_int64


class MegaError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{status_name(status)}: {msg}")
        self.status = status


class mega_csr(_c.Structure):
    _fields_ = [("num_nodes", _c.c_int64), ("num_edges", _c.c_int64), ("indptr", P), ("indices", P)]


class mega_schedule_opts(_c.Structure):
    _fields_ = [("struct_size", _c.c_uint32), ("window", _c.c_int32), ("candidate_cap", _c.c_int32),
                ("order", _c.c_int32), ("seg_edges", _c.c_int32), ("num_parts", _c.c_int32),
                ("seed", _c.c_uint64), ("block_rows", _c.c_int32), ("block_sweeps", _c.c_int32)]


class mega_layout_stats(_c.Structure):
    _fields_ = [("struct_size", _c.c_uint32)] + [(k, _c.c_int64) for k in (
        "num_nodes", "num_edges", "num_parts", "window", "candidate_cap", "seg_edges", "order", "path_length",
        "revisits", "jumps", "tile_unique_sources", "max_in_degree", "max_out_degree")] + [
        ("preprocess_seconds", _c.c_double)] + [(k, _c.c_int64) for k in ("block_rows", "num_blocks",
                                                                          "block_sweeps")]


_VIEW_INTS = ("num_nodes", "num_edges", "row_begin", "row_end", "part_edges", "num_fwd_items", "num_fwd_splits",
              "num_bwd_items", "num_bwd_splits", "num_parts")
_VIEW_PTRS = ("perm", "new_of_old", "bounds", "indptr", "src", "eid", "cindptr", "cdst", "cpos", "csr2csc",
              "fwd_items", "fwd_splits", "bwd_items", "bwd_splits")


class mega_layout_dist_view(_c.Structure):
    _fields_ = [("struct_size", _c.c_uint32)] + [(k, _c.c_int64) for k in (
        "num_local_items", "num_remote_items", "num_splits", "num_slots", "bwd_own_items_begin", "bwd_own_items_end",
        "bwd_own_splits_begin", "bwd_own_splits_end")] + [(k, _c.POINTER(_c.c_int32)) for k in (
        "local_items", "remote_items", "splits")] + [(k, _c.c_int64) for k in (
        "num_send", "num_recv", "full_recv_rows")] + [(k, _c.POINTER(_c.c_int32)) for k in (
        "send_idx", "send_off", "recv_idx", "recv_off")]


class mega_layout_view(_c.Structure):
    _fields_ = [("struct_size", _c.c_uint32)] + [(k, _c.c_int64) for k in _VIEW_INTS] + [
        (k, _c.POINTER(_c.c_int32)) for k in _VIEW_PTRS]


_lib = None


def lib():
    """Load libmega.so (fails loudly if it has not been built)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: build it with "
                              "`python -m paper_conf_icdcs_dengr24_b200.build` (no CPU fallback exists)")
        L = _c.CDLL(LIB_PATH)
        S = _c.c_int
        sig = {
            "mega_abi_version": (_c.c_int, []),
            "mega_status_string": (_c.c_char_p, [S]),
            "mega_last_error": (_c.c_char_p, []),
            "mega_schedule_opts_init": (None, [P]),
            "mega_preprocess": (S, [P, P, P]),
            "mega_layout_destroy": (None, [P]),
            "mega_layout_stats_get": (S, [P, P]),
            "mega_layout_view_get": (S, [P, _c.c_int32, P]),
            "mega_layout_save": (S, [P, _c.c_char_p]),
            "mega_layout_load": (S, [_c.c_char_p, P]),
            "mega_layout_device_bytes": (S, [P, _c.c_int32, P]),
            "mega_layout_bind_device": (S, [P, _c.c_int32, P, _c.c_size_t, P]),
            "mega_gat_workspace_bytes": (S, [P, _c.c_int32, _c.c_int, _c.c_int, S, P, P]),
            "mega_project_fwd": (S, [P, I64, I64, _c.c_int, P, _c.c_int, _c.c_int, P, P, S, P, I64, P, I64, I64, P]),
            "mega_gat_fwd": (S, [P, _c.c_int32, P, I64, P, P, _c.c_int, _c.c_int, S, _c.c_float, _c.c_uint32, P, I64,
                                 P, P, _c.c_size_t, P]),
            "mega_gat_bwd": (S, [P, _c.c_int32, P, I64, P, P, _c.c_int, _c.c_int, S, _c.c_float, _c.c_uint32, P, I64,
                                 P, I64, P, P, I64, P, I64, P, P, P, _c.c_size_t, P]),
            "mega_project_workspace_bytes": (S, [I64, _c.c_int, _c.c_int, _c.c_int, S, P]),
            "mega_project_bwd": (S, [P, I64, I64, _c.c_int, P, _c.c_int, _c.c_int, S, P, I64, P, I64, P, P,
                                     _c.c_size_t, P]),
            "mega_layout_dist_view_get": (S, [P, _c.c_int32, P]),
            "mega_comm_unique_id": (S, [P]),
            "mega_comm_init": (S, [P, _c.c_int, _c.c_int, _c.c_int, P]),
            "mega_comm_init_local": (S, [_c.c_int, P, P]),
            "mega_comm_destroy": (None, [P]),
            "mega_comm_info": (S, [P, P, P, P, P]),
            "mega_gat_dist_workspace_bytes": (S, [P, _c.c_int32, _c.c_int, _c.c_int, S, P, P]),
            "mega_gat_fwd_dist": (S, [P, _c.c_int32, P, P, I64, P, P, _c.c_int, _c.c_int, S, _c.c_float, _c.c_uint32,
                                      P, I64, P, P, _c.c_size_t, P, P]),
            "mega_gat_bwd_dist": (S, [P, _c.c_int32, P, P, I64, P, P, _c.c_int, _c.c_int, S, _c.c_float, _c.c_uint32,
                                      P, I64, P, I64, P, P, I64, P, I64, P, P, P, _c.c_size_t, P, P]),
            "mega_calib_gather": (S, [P, I64, _c.c_int, P, I64, P, I64, P]),
            "mega_band_build": (S, [P, _c.c_int32, _c.c_int32, P]),
            "mega_band_destroy": (None, [P]),
            "mega_band_view_get": (S, [P, P]),
            "mega_band_device_bytes": (S, [P, P]),
            "mega_band_bind_device": (S, [P, P, _c.c_size_t, P]),
            "mega_band_gat_workspace_bytes": (S, [P, _c.c_int, _c.c_int, S, P]),
            "mega_band_gat_fwd": (S, [P, P, I64, P, P, _c.c_int, _c.c_int, S, _c.c_float, _c.c_uint32, P, I64, P, P,
                                      _c.c_size_t, P]),
            "mega_band_gat_bwd": (S, [P, P, I64, P, P, _c.c_int, _c.c_int, S, _c.c_float, P, I64, P, I64, P, P, I64,
                                      P, P, P, _c.c_size_t, P]),
            "mega_gt_fwd": (S, [P, _c.c_int32, P, P, P, I64, _c.c_int, _c.c_int, S, P, I64, P, P, _c.c_size_t, P]),
            "mega_gt_workspace_bytes": (S, [P, _c.c_int32, _c.c_int, _c.c_int, S, P]),
            "mega_gt_bwd": (S, [P, _c.c_int32, P, P, P, I64, _c.c_int, _c.c_int, S, P, I64, P, P, I64, P, P, P, I64,
                                P, _c.c_size_t, P]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def status_name(s):
    return lib().mega_status_string(s).decode()


def _check(status):
    if status != 0:
        raise MegaError(status, lib().mega_last_error().decode())


def mega_abi_version():
    return lib().mega_abi_version()


class Layout:
    """Owns a mega_layout* and the device images bound to it."""

    def __init__(self, handle):
        self._h = _c.c_void_p(handle)
        self._dev = {}

    def __del__(self):
        if getattr(self, "_h", None) and self._h.value and _lib is not None:
            _lib.mega_layout_destroy(self._h)
            self._h = _c.c_void_p(None)

    @property
    def handle(self):
        return self._h

    def stats(self):
        return mega_layout_stats_get(self)

    def view(self, part=0, arrays=True):
        return mega_layout_view_get(self, part, arrays)

    def bind(self, part=0, stream=None):
        return mega_layout_bind_device(self, part, stream)


def mega_preprocess(indptr, indices, window=0, candidate_cap=0, order="traversal", seg_edges=0, num_parts=1,
                    seed=0, block_rows=0, block_sweeps=0) -> Layout:
    indptr = np.ascontiguousarray(indptr, dtype=np.int64)
    indices = np.ascontiguousarray(indices, dtype=np.int32)
    csr = mega_csr(len(indptr) - 1, len(indices), indptr.ctypes.data, indices.ctypes.data)
    o = mega_schedule_opts()
    lib().mega_schedule_opts_init(_c.byref(o))
    o.window, o.candidate_cap, o.seg_edges, o.num_parts, o.seed = window, candidate_cap, seg_edges, num_parts, seed
    o.block_rows, o.block_sweeps = block_rows, block_sweeps
    o.order = ORDERS[order] if isinstance(order, str) else int(order)
    h = _c.c_void_p()
    _check(lib().mega_preprocess(_c.byref(csr), _c.byref(o), _c.byref(h)))
    return Layout(h.value)


def auto_block_rows(row_bytes: int, l2_bytes: int = 126 * 1024 * 1024) -> int:
    """B for L2 blocking: 0.4 of the L2 in gathered rows (R24)."""
    return max(1, int(0.4 * l2_bytes) // max(1, int(row_bytes)))


def mega_layout_stats_get(layout: Layout) -> dict:
    st = mega_layout_stats()
    _check(lib().mega_layout_stats_get(layout.handle, _c.byref(st)))
    return {k: getattr(st, k) for k, _ in mega_layout_stats._fields_ if k != "struct_size"}


def mega_layout_view_get(layout: Layout, part: int = 0, arrays=True) -> dict:
    """Counts of one part and (arrays=True) copies of its host arrays (numpy int32)."""
    v = mega_layout_view()
    _check(lib().mega_layout_view_get(layout.handle, part, _c.byref(v)))
    d = {k: getattr(v, k) for k in _VIEW_INTS}
    if not arrays:
        return d
    n, rows, e = v.num_nodes, v.row_end - v.row_begin, v.part_edges
    sizes = {"perm": n, "new_of_old": n, "bounds": v.num_parts + 1, "indptr": rows + 1, "src": e, "eid": e,
             "cindptr": n + 1, "cdst": e, "cpos": e, "csr2csc": e, "fwd_items": 4 * v.num_fwd_items,
             "fwd_splits": 3 * v.num_fwd_splits, "bwd_items": 4 * v.num_bwd_items,
             "bwd_splits": 3 * v.num_bwd_splits}
    for k in _VIEW_PTRS:
        ptr = getattr(v, k)
        d[k] = np.ctypeslib.as_array(ptr, shape=(sizes[k],)).copy() if sizes[k] > 0 else np.zeros(0, np.int32)
    d["fwd_items"] = d["fwd_items"].reshape(-1, 4)
    d["bwd_items"] = d["bwd_items"].reshape(-1, 4)
    d["fwd_splits"] = d["fwd_splits"].reshape(-1, 3)
    d["bwd_splits"] = d["bwd_splits"].reshape(-1, 3)
    return d


def mega_layout_save(layout: Layout, path: str):
    _check(lib().mega_layout_save(layout.handle, path.encode()))


def mega_layout_load(path: str) -> Layout:
    h = _c.c_void_p()
    _check(lib().mega_layout_load(path.encode(), _c.byref(h)))
    return Layout(h.value)


def mega_layout_device_bytes(layout: Layout, part: int = 0) -> int:
    b = _c.c_size_t()
    _check(lib().mega_layout_device_bytes(layout.handle, part, _c.byref(b)))
    return b.value


def _stream(stream):
    import torch
    s = torch.cuda.current_stream() if stream is None else stream
    return _c.c_void_p(s.cuda_stream)


def _ptr(t):
    return None if t is None else _c.c_void_p(t.data_ptr())


def mega_layout_bind_device(layout: Layout, part: int = 0, stream=None):
    """Allocates the part's device image on the current device (torch) and copies it."""
    import torch
    nbytes = mega_layout_device_bytes(layout, part)
    buf = torch.empty(max(nbytes, 256) + 256, dtype=torch.uint8, device="cuda")
    off = (-buf.data_ptr()) % 256
    view = buf[off:off + max(nbytes, 256)]
    _check(lib().mega_layout_bind_device(layout.handle, part, _c.c_void_p(view.data_ptr()), nbytes, _stream(stream)))
    layout._dev[part] = buf
    return buf


def _dtype_code(t):
    import torch
    if t.dtype == torch.bfloat16:
        return MEGA_BF16
    if t.dtype == torch.float32:
        return MEGA_F32
    raise TypeError(f"unsupported dtype {t.dtype}")


def mega_gat_workspace_bytes(layout: Layout, part: int, heads: int, head_dim: int, dtype: int):
    f, b = _c.c_size_t(), _c.c_size_t()
    _check(lib().mega_gat_workspace_bytes(layout.handle, part, heads, head_dim, dtype, _c.byref(f), _c.byref(b)))
    return f.value, b.value


def mega_project_fwd(x, w, attn_l, attn_r, heads, head_dim, feat, ctx, ctx_n, ctx_row0=0, in_dim=None, stream=None):
    dt = _dtype_code(x)
    _check(lib().mega_project_fwd(_ptr(x), x.stride(0), x.shape[0], in_dim or w.shape[0], _ptr(w), heads, head_dim,
                                  _ptr(attn_l), _ptr(attn_r), dt, _ptr(feat), feat.stride(0), _ptr(ctx), ctx_n,
                                  ctx_row0, _stream(stream)))


def mega_gat_fwd(layout: Layout, part, feat, attn_l, attn_r, heads, head_dim, out, ctx, ws,
                 negative_slope=SLOPE, flags=0, stream=None):
    dt = _dtype_code(feat)
    _check(lib().mega_gat_fwd(layout.handle, part, _ptr(feat), feat.stride(0), _ptr(attn_l), _ptr(attn_r), heads,
                              head_dim, dt, negative_slope, flags, _ptr(out), out.stride(0), _ptr(ctx), _ptr(ws),
                              ws.numel() * ws.element_size(), _stream(stream)))


def mega_gat_bwd(layout: Layout, part, feat, attn_l, attn_r, heads, head_dim, out, grad_out, ctx, grad_feat,
                 grad_attn_l, grad_attn_r, ws, grad_feat_lp=None, negative_slope=SLOPE, flags=0, stream=None):
    dt = _dtype_code(feat)
    _check(lib().mega_gat_bwd(layout.handle, part, _ptr(feat), feat.stride(0), _ptr(attn_l), _ptr(attn_r), heads,
                              head_dim, dt, negative_slope, flags, _ptr(out), out.stride(0), _ptr(grad_out),
                              grad_out.stride(0), _ptr(ctx), _ptr(grad_feat), grad_feat.stride(0),
                              _ptr(grad_feat_lp), grad_feat_lp.stride(0) if grad_feat_lp is not None else 0,
                              _ptr(grad_attn_l), _ptr(grad_attn_r), _ptr(ws), ws.numel() * ws.element_size(),
                              _stream(stream)))


def mega_project_workspace_bytes(rows, in_dim, heads, head_dim, dtype) -> int:
    b = _c.c_size_t()
    _check(lib().mega_project_workspace_bytes(rows, in_dim, heads, head_dim, dtype, _c.byref(b)))
    return b.value


def mega_project_bwd(x, w, heads, head_dim, grad_feat, grad_w, grad_x=None, in_dim=None, ws=None, stream=None):
    dt = _dtype_code(x)
    _check(lib().mega_project_bwd(_ptr(x), x.stride(0), x.shape[0], in_dim or w.shape[0], _ptr(w), heads, head_dim,
                                  dt, _ptr(grad_feat), grad_feat.stride(0), _ptr(grad_x),
                                  grad_x.stride(0) if grad_x is not None else 0, _ptr(grad_w), _ptr(ws),
                                  0 if ws is None else ws.numel() * ws.element_size(), _stream(stream)))


def mega_calib_gather(table, row_bytes, idx, sink, stream=None):
    """Measurement helper: gather rows idx of `table` (device, [rows][row_bytes])."""
    _check(lib().mega_calib_gather(_ptr(table), table.numel() * table.element_size() // row_bytes, row_bytes,
                                   _ptr(idx), idx.numel(), _ptr(sink), sink.numel(), _stream(stream)))


# ---------------- k GPUs (include/mega.h "k GPUs: destination partitions") ----------------
def mega_layout_dist_view_get(layout: Layout, part: int = 0) -> dict:
    """Host copy of the k-GPU work split of one part (local / remote forward items, merge records,
    own-source ranges of the backward items)."""
    v = mega_layout_dist_view()
    _check(lib().mega_layout_dist_view_get(layout.handle, part, _c.byref(v)))
    d = {k: getattr(v, k) for k, _ in mega_layout_dist_view._fields_[1:9]}
    d.update({k: getattr(v, k) for k in ("num_send", "num_recv", "full_recv_rows")})
    for k, w, n in (("local_items", 4, v.num_local_items), ("remote_items", 4, v.num_remote_items),
                    ("splits", 3, v.num_splits)):
        ptr = getattr(v, k)
        d[k] = (np.ctypeslib.as_array(ptr, shape=(n * w,)).copy() if n > 0 else np.zeros(0, np.int32)).reshape(-1, w)
    k1 = layout.view(part, arrays=False)["num_parts"] + 1
    for k, n in (("send_idx", v.num_send), ("recv_idx", v.num_recv), ("send_off", k1 if k1 > 2 else 0),
                 ("recv_off", k1 if k1 > 2 else 0)):
        ptr = getattr(v, k)
        d[k] = np.ctypeslib.as_array(ptr, shape=(n,)).copy() if n > 0 and ptr else np.zeros(0, np.int32)
    return d


class Comm:
    """Owns a mega_comm* (library-owned communicator)."""

    def __init__(self, handle):
        self._h = _c.c_void_p(handle)

    def __del__(self):
        if getattr(self, "_h", None) and self._h.value and _lib is not None:
            _lib.mega_comm_destroy(self._h)
            self._h = _c.c_void_p(None)

    @property
    def handle(self):
        return self._h

    def info(self):
        a, b, c, d = _c.c_int(), _c.c_int(), _c.c_int(), _c.c_int()
        _check(lib().mega_comm_info(self._h, _c.byref(a), _c.byref(b), _c.byref(c), _c.byref(d)))
        return {"nranks": a.value, "rank": b.value, "device": c.value, "transport": ("nccl", "local")[d.value]}


def mega_comm_unique_id() -> bytes:
    buf = (_c.c_uint8 * 128)()
    _check(lib().mega_comm_unique_id(buf))
    return bytes(buf)


def mega_comm_init(uid: bytes, nranks: int, rank: int, device: int) -> Comm:
    assert len(uid) == 128
    buf = (_c.c_uint8 * 128).from_buffer_copy(uid)
    h = _c.c_void_p()
    _check(lib().mega_comm_init(buf, nranks, rank, device, _c.byref(h)))
    return Comm(h.value)


def mega_comm_init_local(nranks: int, devices=None):
    """LOCAL transport: all ranks in this process -> list of Comm."""
    out = (_c.c_void_p * nranks)()
    devs = None if devices is None else (_c.c_int * nranks)(*devices)
    _check(lib().mega_comm_init_local(nranks, devs, out))
    return [Comm(out[r]) for r in range(nranks)]


def mega_gat_dist_workspace_bytes(layout: Layout, part: int, heads: int, head_dim: int, dtype: int):
    f, b = _c.c_size_t(), _c.c_size_t()
    _check(lib().mega_gat_dist_workspace_bytes(layout.handle, part, heads, head_dim, dtype, _c.byref(f),
                                               _c.byref(b)))
    return f.value, b.value


def mega_gat_fwd_dist(layout: Layout, part, comm: Comm, feat, attn_l, attn_r, heads, head_dim, out, ctx, ws,
                      negative_slope=SLOPE, flags=0, stream=None, comm_stream=None):
    dt = _dtype_code(feat)
    _check(lib().mega_gat_fwd_dist(layout.handle, part, comm.handle, _ptr(feat), feat.stride(0), _ptr(attn_l),
                                   _ptr(attn_r), heads, head_dim, dt, negative_slope, flags, _ptr(out), out.stride(0),
                                   _ptr(ctx), _ptr(ws), ws.numel() * ws.element_size(), _stream(stream),
                                   _stream(comm_stream)))


def mega_gat_bwd_dist(layout: Layout, part, comm: Comm, feat, attn_l, attn_r, heads, head_dim, out, grad_out, ctx,
                      grad_feat, grad_attn_l, grad_attn_r, ws, grad_feat_lp=None, negative_slope=SLOPE, flags=0,
                      stream=None, comm_stream=None):
    dt = _dtype_code(feat)
    _check(lib().mega_gat_bwd_dist(layout.handle, part, comm.handle, _ptr(feat), feat.stride(0), _ptr(attn_l),
                                   _ptr(attn_r), heads, head_dim, dt, negative_slope, flags, _ptr(out), out.stride(0),
                                   _ptr(grad_out), grad_out.stride(0), _ptr(ctx), _ptr(grad_feat),
                                   grad_feat.stride(0), _ptr(grad_feat_lp),
                                   grad_feat_lp.stride(0) if grad_feat_lp is not None else 0, _ptr(grad_attn_l),
                                   _ptr(grad_attn_r), _ptr(ws), ws.numel() * ws.element_size(), _stream(stream),
                                   _stream(comm_stream)))


# NEXT-3: Graph Transformer edge attention (include/mega.h mega_gt_*; fp32 or bf16 storage)
def mega_gt_workspace_bytes(layout: Layout, part: int, heads: int, head_dim: int = 0, dtype: int = MEGA_F32):
    b = _c.c_size_t()
    _check(lib().mega_gt_workspace_bytes(layout.handle, part, heads, head_dim or 1, dtype, _c.byref(b)))
    return b.value


def _gt_check(name, tensors, ld_group, dtype):
    """mega_gt_* take row-major operands of one dtype with ONE leading dimension per group:
    refuse anything else instead of letting the kernels read it as the wrong data."""
    for t in tensors:
        if t.dtype != dtype or not t.is_cuda or t.dim() != 2 or t.stride(1) != 1:
            raise TypeError(f"{name}: operands must be {dtype} CUDA 2-D tensors with unit column stride")
    if len({t.stride(0) for t in ld_group}) != 1:
        raise ValueError(f"{name}: {len(ld_group)} operands sharing one leading dimension have different strides")


def mega_gt_fwd(layout: Layout, part, q, k, v, heads, head_dim, out, lse, ws=None, stream=None):
    import torch
    _gt_check("mega_gt_fwd", (q, k, v, out), (q, k, v), q.dtype)
    _gt_check("mega_gt_fwd", (lse,), (lse,), torch.float32)
    _check(lib().mega_gt_fwd(layout.handle, part, _ptr(q), _ptr(k), _ptr(v), q.stride(0), heads, head_dim,
                             _dtype_code(q), _ptr(out), out.stride(0), _ptr(lse), _ptr(ws),
                             0 if ws is None else ws.numel() * ws.element_size(), _stream(stream)))


def mega_gt_bwd(layout: Layout, part, q, k, v, heads, head_dim, out, lse, grad_out, grad_q, grad_k, grad_v, ws,
                stream=None):
    import torch
    _gt_check("mega_gt_bwd", (q, k, v, out, grad_out), (q, k, v), q.dtype)
    _gt_check("mega_gt_bwd", (lse, grad_q, grad_k, grad_v), (grad_q, grad_k, grad_v), torch.float32)
    _check(lib().mega_gt_bwd(layout.handle, part, _ptr(q), _ptr(k), _ptr(v), q.stride(0), heads, head_dim,
                             _dtype_code(q), _ptr(out), out.stride(0), _ptr(lse), _ptr(grad_out), grad_out.stride(0),
                             _ptr(grad_q), _ptr(grad_k), _ptr(grad_v), grad_k.stride(0), _ptr(ws),
                             ws.numel() * ws.element_size(), _stream(stream)))


# ---------------- NEXT-2: the faithful path-band layout (include/mega.h) ----------------
class mega_band_view(_c.Structure):
    _fields_ = [("struct_size", _c.c_uint32), ("num_nodes", _c.c_int64), ("num_edges", _c.c_int64),
                ("length", _c.c_int64), ("window", _c.c_int32), ("cap", _c.c_int32), ("jumps", _c.c_int64),
                ("virtual_edges", _c.c_int64), ("edges_u", _c.c_int64), ("num_slots", _c.c_int64),
                ("num_merges", _c.c_int64), ("build_seconds", _c.c_double), ("P", P), ("own", P), ("lmask", P),
                ("rmask", P), ("cptr", P), ("cnt", P), ("slot", P), ("merges", P)]


class Band:
    """Owns a mega_band* and its device image."""

    def __init__(self, handle):
        self._h = _c.c_void_p(handle)
        self._dev = None

    def __del__(self):
        if getattr(self, "_h", None) and self._h.value and _lib is not None:
            _lib.mega_band_destroy(self._h)
            self._h = _c.c_void_p(None)

    @property
    def handle(self):
        return self._h

    def view(self):
        v = mega_band_view()
        v.struct_size = _c.sizeof(mega_band_view)
        _check(lib().mega_band_view_get(self._h, _c.byref(v)))
        L = v.length
        d = {k: getattr(v, k) for k, _ in mega_band_view._fields_[1:12]}

        def arr(ptr, n, dt):
            if n == 0 or not ptr:
                return np.zeros(0, dt)
            return np.ctypeslib.as_array(_c.cast(ptr, _c.POINTER(np.ctypeslib.as_ctypes_type(dt))), (n,)).copy()
        d["P"] = arr(v.P, L, np.int32)
        d["own"] = arr(v.own, L, np.uint64)
        d["lmask"] = arr(v.lmask, L, np.uint64)
        d["rmask"] = arr(v.rmask, L, np.uint64)
        d["cptr"] = arr(v.cptr, L + 1, np.int32)
        d["cnt"] = arr(v.cnt, int(d["cptr"][-1]) if L else 0, np.uint16)
        d["slot"] = arr(v.slot, L, np.int32)
        d["merges"] = arr(v.merges, 3 * v.num_merges, np.int32).reshape(-1, 3)
        return d

    def bind(self, stream=None):
        import torch
        nb = _c.c_size_t()
        _check(lib().mega_band_device_bytes(self._h, _c.byref(nb)))
        n = max(nb.value, 256)
        buf = torch.empty(n + 256, dtype=torch.uint8, device="cuda")
        off = (-buf.data_ptr()) % 256
        _check(lib().mega_band_bind_device(self._h, _c.c_void_p(buf.data_ptr() + off), nb.value, _stream(stream)))
        self._dev = buf
        return buf


def mega_band_build(indptr, indices, window=0, cap=0) -> Band:
    indptr = np.ascontiguousarray(indptr, dtype=np.int64)
    indices = np.ascontiguousarray(indices, dtype=np.int32)
    csr = mega_csr(len(indptr) - 1, len(indices), indptr.ctypes.data, indices.ctypes.data)
    h = _c.c_void_p()
    _check(lib().mega_band_build(_c.byref(csr), window, cap, _c.byref(h)))
    return Band(h.value)


def mega_band_gat_workspace_bytes(band: Band, heads: int, head_dim: int, dtype: int) -> int:
    w = _c.c_size_t()
    _check(lib().mega_band_gat_workspace_bytes(band.handle, heads, head_dim, dtype, _c.byref(w)))
    return w.value


def mega_band_gat_fwd(band: Band, feat, attn_l, attn_r, heads, head_dim, out, ctx, ws, negative_slope=SLOPE,
                      flags=0, stream=None):
    dt = _dtype_code(feat)
    _check(lib().mega_band_gat_fwd(band.handle, _ptr(feat), feat.stride(0), _ptr(attn_l), _ptr(attn_r), heads,
                                   head_dim, dt, negative_slope, flags, _ptr(out), out.stride(0), _ptr(ctx), _ptr(ws),
                                   ws.numel() * ws.element_size(), _stream(stream)))


def mega_band_gat_bwd(band: Band, feat, attn_l, attn_r, heads, head_dim, out, grad_out, ctx, grad_feat, grad_attn_l,
                      grad_attn_r, ws, negative_slope=SLOPE, stream=None):
    dt = _dtype_code(feat)
    _check(lib().mega_band_gat_bwd(band.handle, _ptr(feat), feat.stride(0), _ptr(attn_l), _ptr(attn_r), heads,
                                   head_dim, dt, negative_slope, _ptr(out), out.stride(0), _ptr(grad_out),
                                   grad_out.stride(0), _ptr(ctx), _ptr(grad_feat), grad_feat.stride(0),
                                   _ptr(grad_attn_l), _ptr(grad_attn_r), _ptr(ws), ws.numel() * ws.element_size(),
                                   _stream(stream)))
