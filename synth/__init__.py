"""mega-synth v1: seeded synthetic inputs shared by oracle/, tests/ and bench.py.

Test infrastructure with none of the method's arithmetic: it only draws graphs
(CSR by destination, int64 indptr / int32 source indices) and numbers.  The
recipe is stated in DESIGN.md ("Input recipe"); the five workload shapes are
BASELINE.json's `configs` (node/edge counts, feature widths, heads x hidden).
The homophily mu, exponent gamma and max-degree d_cap are public-dataset
figures used only to shape the synthetic graphs; they do
not come from the paper.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "csrc", "mega_synth.c")
_LIB = os.path.join(_HERE, "libmegasynth.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile the generator (plain C, gcc -O2 -fopenmp)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-std=c11",
                               "-o", _LIB, _SRC, "-lm"])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.msynth_graph.restype = ctypes.c_int
        lib.msynth_graph.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int, ctypes.c_int32,
                                     ctypes.c_double, ctypes.c_double, ctypes.c_double, ctypes.c_uint64,
                                     ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p]
        lib.msynth_normal_f32.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_float, ctypes.c_void_p]
        lib.msynth_uniform_f32.argtypes = [ctypes.c_uint64, ctypes.c_int64, ctypes.c_float, ctypes.c_float,
                                           ctypes.c_void_p]
        lib.msynth_draw.restype = ctypes.c_uint64
        lib.msynth_draw.argtypes = [ctypes.c_uint64, ctypes.c_uint64]
        _lib = lib
    return _lib


@dataclass(frozen=True)
class GraphConfig:
    name: str
    index: int            # position in BASELINE.json configs (seed = 0x4D454741 + 16*index)
    n: int
    m: int                # directed edge count (both directions counted, Table II)
    directed: bool
    f_in: int
    heads: int
    head_dim: int
    layers: int
    communities: int
    mu: float
    gamma: float
    d_cap: float
    batch: str = ""       # Table II dataset shape of a block-diagonal batch (synth/batch.py), "" = one graph
    num_graphs: int = 0
    drop: float = 0.0     # edge-dropping fraction per graph

    @property
    def f_in_pad(self) -> int:    # 16-byte rows for bf16 (TMA/ld.128): multiple of 8
        return (self.f_in + 7) // 8 * 8

    @property
    def dim(self) -> int:
        return self.heads * self.head_dim

    @property
    def seed(self) -> int:
        return 0x4D454741 + 16 * self.index


# BASELINE.json "configs", in order.
CONFIGS = {
    "cora": GraphConfig("cora", 0, 2708, 10556, False, 1433, 8, 8, 1, 7, 0.81, 2.5, 170),
    "pubmed": GraphConfig("pubmed", 1, 19717, 88648, False, 500, 8, 8, 1, 3, 0.80, 2.5, 170),
    "arxiv": GraphConfig("arxiv", 2, 169343, 1166243, True, 128, 4, 64, 3, 40, 0.65, 2.2, 13000),
    "reddit": GraphConfig("reddit", 3, 232965, 114615892, False, 602, 4, 64, 1, 41, 0.78, 2.1, 21000),
    "products": GraphConfig("products", 4, 2449029, 61859140, False, 100, 4, 128, 3, 47, 0.81, 2.3, 17000),
}


# The paper's own workload: batches of small graphs, hidden 128 = 8 heads x 16
# (batch 64 / hidden 128; batch 64, 128, 256; 20% edge drop).
# n and m are filled in from the generated batch by get_config().
_BATCHES = {
    "zinc-b64": ("zinc", 64, 0.0), "zinc-b128": ("zinc", 128, 0.0), "zinc-b256": ("zinc", 256, 0.0),
    "aqsol-b128": ("aqsol", 128, 0.0), "aqsol-b128-drop20": ("aqsol", 128, 0.2),
    "csl-b128": ("csl", 128, 0.0), "cycles-b128": ("cycles", 128, 0.0),
}


def _batch_graph(name, num_graphs, drop, seed):
    from synth.batch import drop_edges, make_batch
    ip, ix, gptr = make_batch(name, num_graphs, seed)
    if drop > 0:
        ip, ix = drop_edges(ip, ix, gptr, drop, seed + 1)
    return ip, ix, gptr


def get_config(name: str) -> GraphConfig:
    """BASELINE.json configs by name, or a batch config (exact n, m of its seeded batch)."""
    if name in CONFIGS:
        return CONFIGS[name]
    ds, b, drop = _BATCHES[name]
    index = 5 + sorted(_BATCHES).index(name)
    seed = 0x4D454741 + 16 * index
    ip, ix, _ = _batch_graph(ds, b, drop, seed)
    return GraphConfig(name, index, len(ip) - 1, len(ix), False, 128, 8, 16, 4, 0, 0.0, 0.0, 0.0,
                       batch=ds, num_graphs=b, drop=drop)


def scaled(cfg: GraphConfig, n: int, m: int, name: str | None = None) -> GraphConfig:
    """Same shape recipe at a smaller size (for tests)."""
    if not cfg.directed and m % 2:
        m += 1
    return GraphConfig(name or f"{cfg.name}-{n}", cfg.index, n, m, cfg.directed, cfg.f_in, cfg.heads,
                       cfg.head_dim, cfg.layers, cfg.communities, cfg.mu, cfg.gamma,
                       min(cfg.d_cap, max(8.0, 0.3 * n)))


def make_graph(cfg: GraphConfig):
    """-> (indptr int64[n+1], indices int32[m], stats dict).  Rows are destinations."""
    if cfg.batch:
        ip, ix, _ = _batch_graph(cfg.batch, cfg.num_graphs, cfg.drop, cfg.seed)
        return ip, ix, {"duplicates": 0, "self_loops": 0}
    lib = _load()
    indptr = np.empty(cfg.n + 1, dtype=np.int64)
    indices = np.empty(cfg.m, dtype=np.int32)
    st = np.zeros(2, dtype=np.int64)
    rc = lib.msynth_graph(cfg.n, cfg.m, int(cfg.directed), cfg.communities, cfg.mu, cfg.gamma, cfg.d_cap,
                          cfg.seed, indptr.ctypes.data, indices.ctypes.data, st.ctypes.data)
    if rc != 0:
        raise ValueError(f"msynth_graph rejected {cfg}")
    return indptr, indices, {"duplicates": int(st[0]), "self_loops": int(st[1])}


def communities(cfg: GraphConfig) -> np.ndarray:
    """Community id of every node of make_graph(cfg) (the generator's own assignment,
    comm[v] = draw(seed ^ 0x2222..., v) % C; used only for the community-sorted
    upper-bound ablation order of bench.py)."""
    if cfg.batch:
        raise ValueError("batch workloads have no community structure")
    M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
    with np.errstate(over="ignore"):
        z = (np.uint64(cfg.seed ^ 0x2222222222222222) +
             (np.arange(cfg.n, dtype=np.uint64) + np.uint64(1)) * np.uint64(0x9E3779B97F4A7C15)) & M64
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return (z % np.uint64(cfg.communities)).astype(np.int32)


def relabel(indptr, indices, order):
    """The same graph with node order[r] renamed r (rows permuted, sources renamed)."""
    indptr = np.asarray(indptr, np.int64)
    order = np.asarray(order, np.int64)
    n = len(indptr) - 1
    new_of = np.empty(n, np.int64)
    new_of[order] = np.arange(n)
    deg = np.diff(indptr)[order]
    ip2 = np.zeros(n + 1, np.int64)
    np.cumsum(deg, out=ip2[1:])
    pos = np.repeat(indptr[order] - ip2[:-1], deg) + np.arange(ip2[-1])
    return ip2, new_of[np.asarray(indices)[pos]].astype(np.int32)


def normal(seed: int, shape, scale: float = 1.0) -> np.ndarray:
    lib = _load()
    out = np.empty(int(np.prod(shape)), dtype=np.float32)
    lib.msynth_normal_f32(seed & 0xFFFFFFFFFFFFFFFF, out.size, scale, out.ctypes.data)
    return out.reshape(shape)


def uniform(seed: int, shape, lo: float, hi: float) -> np.ndarray:
    lib = _load()
    out = np.empty(int(np.prod(shape)), dtype=np.float32)
    lib.msynth_uniform_f32(seed & 0xFFFFFFFFFFFFFFFF, out.size, lo, hi, out.ctypes.data)
    return out.reshape(shape)


def _sub(cfg_seed: int, stream: int, layer: int = 0) -> int:
    return (cfg_seed + stream) ^ (layer << 40)


def make_layer_inputs(cfg: GraphConfig, layer: int = 0, in_dim: int | None = None):
    """fp32 X [n, in_pad] (pad columns 0), W [in_pad, D] (pad rows 0), a_l, a_r [H, F],
    grad_out [n, D].  Sub-streams: +1 X, +2 W, +3 a_l, +4 a_r, +5 grad_out."""
    f_in = cfg.f_in if in_dim is None else in_dim
    f_pad = (f_in + 7) // 8 * 8
    D, H, F = cfg.dim, cfg.heads, cfg.head_dim
    x = np.zeros((cfg.n, f_pad), dtype=np.float32)
    x[:, :f_in] = normal(_sub(cfg.seed, 1, layer), (cfg.n, f_in))
    lim = float(np.sqrt(6.0 / (f_in + D)))
    w = np.zeros((f_pad, D), dtype=np.float32)
    w[:f_in] = uniform(_sub(cfg.seed, 2, layer), (f_in, D), -lim, lim)
    a_l = normal(_sub(cfg.seed, 3, layer), (H, F), float(1.0 / np.sqrt(F)))
    a_r = normal(_sub(cfg.seed, 4, layer), (H, F), float(1.0 / np.sqrt(F)))
    g = normal(_sub(cfg.seed, 5, layer), (cfg.n, D))
    return {"x": x, "w": w, "a_l": a_l, "a_r": a_r, "grad_out": g, "in_dim": f_in}


def bf16_round(a: np.ndarray) -> np.ndarray:
    """Round fp32 values to bf16 (round-to-nearest-even), returned as fp32 values."""
    a = np.ascontiguousarray(a, dtype=np.float32)
    u = a.view(np.uint32).astype(np.uint64)
    r = ((u + 0x7FFF + ((u >> 16) & 1)) >> 16) << 16
    return r.astype(np.uint32).view(np.float32).reshape(a.shape)


from .tiny import random_multigraph, from_edge_list, to_edge_list  # noqa: E402,F401
