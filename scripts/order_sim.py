"""Offline comparison of node orders by simulated L2 misses (analysis only).

For each order, the forward gather stream (sources of the relabelled CSR in
row order) goes through a fully associative LRU of `cap` rows; fewer misses =
less HBM traffic for the row gathers.  Usage: python scripts/order_sim.py [config]
"""
import ctypes
import os
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
from paper_conf_icdcs_dengr24_b200 import mega as M  # noqa: E402

HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.path.join(HERE, "liblrusim.so")
subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-o", SO, os.path.join(HERE, "lru_sim.c")])
lib = ctypes.CDLL(SO)
lib.lru_misses.restype = ctypes.c_int64
lib.lru_misses.argtypes = [ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64]


def stream_of(perm, ip, ix):
    """sources (new ids) in new-row order."""
    n = len(perm)
    new = np.empty(n, np.int64)
    new[perm] = np.arange(n)
    deg = np.diff(ip)
    rows = perm.astype(np.int64)
    starts = ip[rows]
    lens = deg[rows]
    idx = np.repeat(starts - np.cumsum(np.r_[0, lens[:-1]]), lens) + np.arange(lens.sum())
    return new[ix[idx]].astype(np.int32)


def communities(cfg):
    lib_s = synth._load()
    s_comm = (cfg.seed ^ 0x2222222222222222) & 0xFFFFFFFFFFFFFFFF
    return np.array([lib_s.msynth_draw(s_comm, v) % cfg.communities for v in range(cfg.n)], np.int64)


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "products"
    caps = [int(c) for c in (sys.argv[2].split(",") if len(sys.argv) > 2 else ["32768", "65536", "100000"])]
    cfg = synth.CONFIGS[name]
    ip, ix, _ = synth.make_graph(cfg)
    n, m = cfg.n, cfg.m
    orders = {}
    for nm, kw in [("identity", dict(order="identity")), ("traversal", dict(order="traversal")),
                   ("degree", dict(order="degree")), ("blocked", dict(order="traversal", block_rows=51814))]:
        t = time.time()
        lay = M.mega_preprocess(ip, ix, **kw)
        orders[nm] = lay.view(0)["perm"].astype(np.int64)
        print(f"{nm}: preprocess {time.time() - t:.1f}s", flush=True)
        del lay
    comm = communities(cfg)
    pos = np.empty(n, np.int64)
    pos[orders["traversal"]] = np.arange(n)
    orders["community+traversal"] = np.lexsort((pos, comm))
    extra = os.environ.get("ORDER_NPY")
    if extra:
        orders["extra"] = np.load(extra)
    for nm, perm in orders.items():
        s = stream_of(perm, ip, ix)
        res = []
        for cap in caps:
            mi = lib.lru_misses(n, s.ctypes.data, len(s), cap)
            res.append(f"cap {cap}: miss {mi / m:.3f}")
        print(f"{nm:22s} " + "  ".join(res), flush=True)


if __name__ == "__main__":
    main()
