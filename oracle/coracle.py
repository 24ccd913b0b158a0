"""ctypes loader for oracle/c/oracle.c — TEST INFRASTRUCTURE ONLY (see __init__).

Same definitions as oracle/gat.py and oracle/traverse.py, for sizes numpy
cannot reach in seconds.  Inputs are the stored values (fp32 or bf16-rounded
fp32), computed on in fp64.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from .gat import SLOPE

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "c", "oracle.c")
_LIB = os.path.join(_HERE, "c", "liboracle.so")
_lib = None
P = ctypes.c_void_p
I64 = ctypes.c_int64


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11", "-o", _LIB, _SRC, "-lm"])
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        L.ora_gat_fwd.argtypes = [I64, P, P, ctypes.c_int, ctypes.c_int, P, P, P, ctypes.c_double, P, P, P, P]
        L.ora_gat_fwd_rows.argtypes = [I64, P, P, ctypes.c_int, ctypes.c_int, P, P, P, ctypes.c_double, I64, P,
                                       P, P]
        L.ora_gat_bwd.argtypes = [I64, P, P, ctypes.c_int, ctypes.c_int, P, P, P, ctypes.c_double, P, P, P, P, P,
                                  P, P, P, P, P]
        L.ora_gat_bwd_srcs.argtypes = [I64, P, P, ctypes.c_int, ctypes.c_int, P, P, P, ctypes.c_double, P, I64,
                                       P, P]
        L.ora_traverse.argtypes = [I64, P, P, ctypes.c_int, ctypes.c_int, P, P, P]
        L.ora_traverse.restype = ctypes.c_int
        L.ora_l2_blocks.argtypes = [I64, P, P, ctypes.c_int32, ctypes.c_int, P, P]
        L.ora_l2_blocks.restype = ctypes.c_int
        _lib = L
    return _lib


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def _graph(indptr, indices):
    return np.ascontiguousarray(indptr, np.int64), np.ascontiguousarray(indices, np.int32)


def gat_forward(indptr, indices, Wh, a_l, a_r, slope=SLOPE):
    """Wh: [n, H, F] (float32 values).  -> dict(out [n,H,F], lse, el, er [n,H]) fp64."""
    ip, ix = _graph(indptr, indices)
    Wh = _f32(Wh)
    n, H, F = Wh.shape
    a_l, a_r = _f32(a_l), _f32(a_r)
    out = np.empty((n, H, F)); lse = np.empty((n, H)); el = np.empty((n, H)); er = np.empty((n, H))
    lib().ora_gat_fwd(n, ip.ctypes.data, ix.ctypes.data, H, F, Wh.ctypes.data, a_l.ctypes.data, a_r.ctypes.data,
                      slope, out.ctypes.data, lse.ctypes.data, el.ctypes.data, er.ctypes.data)
    return {"out": out, "lse": lse, "el": el, "er": er}


def gat_forward_rows(indptr, indices, Wh, a_l, a_r, rows, slope=SLOPE):
    ip, ix = _graph(indptr, indices)
    Wh = _f32(Wh)
    n, H, F = Wh.shape
    a_l, a_r = _f32(a_l), _f32(a_r)
    rows = np.ascontiguousarray(rows, np.int64)
    out = np.empty((len(rows), H, F)); lse = np.empty((len(rows), H))
    lib().ora_gat_fwd_rows(n, ip.ctypes.data, ix.ctypes.data, H, F, Wh.ctypes.data, a_l.ctypes.data,
                           a_r.ctypes.data, slope, len(rows), rows.ctypes.data, out.ctypes.data, lse.ctypes.data)
    return {"out": out, "lse": lse}


def gat_backward(indptr, indices, Wh, a_l, a_r, grad_out, slope=SLOPE, fwd=None):
    ip, ix = _graph(indptr, indices)
    Wh = _f32(Wh)
    n, H, F = Wh.shape
    a_l, a_r, g = _f32(a_l), _f32(a_r), _f32(grad_out)
    if fwd is None:
        fwd = gat_forward(ip, ix, Wh, a_l, a_r, slope)
    out = np.ascontiguousarray(fwd["out"], np.float64)
    lse = np.ascontiguousarray(fwd["lse"], np.float64)
    el = np.ascontiguousarray(fwd["el"], np.float64)
    er = np.ascontiguousarray(fwd["er"], np.float64)
    gf = np.empty((n, H, F)); gal = np.empty((H, F)); gar = np.empty((H, F))
    dl = np.empty((n, H)); dr = np.empty((n, H))
    lib().ora_gat_bwd(n, ip.ctypes.data, ix.ctypes.data, H, F, Wh.ctypes.data, a_l.ctypes.data, a_r.ctypes.data,
                      slope, g.ctypes.data, out.ctypes.data, lse.ctypes.data, el.ctypes.data, er.ctypes.data,
                      gf.ctypes.data, gal.ctypes.data, gar.ctypes.data, dl.ctypes.data, dr.ctypes.data)
    return {"grad_feat": gf, "grad_attn_l": gal, "grad_attn_r": gar, "del": dl, "der": dr}


def gat_backward_srcs(indptr, indices, Wh, a_l, a_r, grad_out, srcs, slope=SLOPE):
    ip, ix = _graph(indptr, indices)
    Wh = _f32(Wh)
    n, H, F = Wh.shape
    a_l, a_r, g = _f32(a_l), _f32(a_r), _f32(grad_out)
    srcs = np.ascontiguousarray(srcs, np.int64)
    gf = np.empty((len(srcs), H, F))
    lib().ora_gat_bwd_srcs(n, ip.ctypes.data, ix.ctypes.data, H, F, Wh.ctypes.data, a_l.ctypes.data,
                           a_r.ctypes.data, slope, g.ctypes.data, len(srcs), srcs.ctypes.data, gf.ctypes.data)
    return gf


def traverse(n, indptr, indices, window=0, cap=0, with_path=True):
    ip, ix = _graph(indptr, indices)
    perm = np.empty(max(n, 1), np.int32)
    Pbuf = np.empty(2 * n + 2, np.int32) if with_path else None
    st = np.zeros(4, np.int64)
    lib().ora_traverse(n, ip.ctypes.data, ix.ctypes.data, window, cap, perm.ctypes.data,
                       Pbuf.ctypes.data if with_path else None, st.ctypes.data)
    res = {"perm": perm[:n], "path_length": int(st[0]), "jumps": int(st[1]), "window": int(st[2]),
           "cap": int(st[3])}
    if with_path:
        res["P"] = Pbuf[:st[0]].copy()
    return res


def l2_blocks(indptr, indices, B, sweeps=0):
    """-> (label int32 [n], sweeps run); same definition as oracle/blocks.propagate."""
    ip, ix = _graph(indptr, indices)
    n = len(ip) - 1
    label = np.empty(n, np.int32)
    st = np.zeros(1, np.int64)
    lib().ora_l2_blocks(n, ip.ctypes.data, ix.ctypes.data, int(B), int(sweeps), label.ctypes.data, st.ctypes.data)
    return label, int(st[0])
