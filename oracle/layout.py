"""The exact relabelled layout — plain numpy definition. Integer only.

Test infrastructure only (see oracle/__init__.py).

MEGA lays node embeddings out in the order the traversal visits them
("graph vertexes are sorted according to the order they are
accessed").  Because the north_star requires the edge multiset
to be preserved exactly, we keep every edge in a relabelled CSR instead of the
paper's band with virtual edges (R20):

  (i)   row r holds the in-edges of old node perm[r]; each input edge position
        e maps to (new_of_old[src_e], e); rows sorted ascending by that pair;
  (ii)  per part, a CSC: stable sort of the part's CSR positions by source;
        cdst = local destination row, cpos = CSR position, csr2csc = cpos^-1;
  (iii) work items: one item per row; a row with more than S edges is split
        into ceil(deg/S) segments, each owning a partial-state slot;
  (iv)  k edge-balanced contiguous partitions (the exact form of "adjacent
        path partitions"): b_0 = 0,
        b_p = min{r : indptr'[r] >= ceil(p*m/k)}, b_k = n.
"""
from __future__ import annotations

import numpy as np

def auto_seg_edges(m: int) -> int:
    """S = 256 (a layout input like the tile sizes)."""
    return 256


def relabel(indptr, indices, perm):
    """(i): -> new_of_old, indptr', src', eid' (int64)."""
    indptr = np.asarray(indptr, np.int64)
    n = len(indptr) - 1
    perm = np.asarray(perm, np.int64)
    new_of_old = np.empty(n, np.int64)
    new_of_old[perm] = np.arange(n)
    deg = np.diff(indptr)
    dst_old = np.repeat(np.arange(n), deg)
    src_old = np.asarray(indices, np.int64)
    new_dst = new_of_old[dst_old]
    new_src = new_of_old[src_old]
    eid = np.arange(len(src_old), dtype=np.int64)
    order = np.lexsort((eid, new_src, new_dst))
    ip = np.zeros(n + 1, np.int64)
    ip[1:] = np.cumsum(np.bincount(new_dst, minlength=n))
    return new_of_old, ip, new_src[order], eid[order]


def partition_bounds(indptr_new, k: int):
    """(iv): b_p = min{r : indptr'[r] >= ceil(p*m/k)}."""
    n = len(indptr_new) - 1
    m = int(indptr_new[-1])
    b = [0]
    for p in range(1, k):
        t = -(-p * m // k)
        b.append(int(np.searchsorted(indptr_new, t, side="left")))
    b.append(n)
    return np.asarray(b, np.int64)


def items(indptr_local, S: int):
    """(iii): -> items [nitems, 4] = (row, e_begin, e_end, slot or -1),
    splits [nsplit, 3] = (row, first_slot, nseg)."""
    it, sp = [], []
    slot = 0
    for r in range(len(indptr_local) - 1):
        b, e = int(indptr_local[r]), int(indptr_local[r + 1])
        if e - b <= S:
            it.append((r, b, e, -1))
        else:
            nseg = -(-(e - b) // S)
            sp.append((r, slot, nseg))
            for k in range(nseg):
                it.append((r, b + k * S, min(e, b + (k + 1) * S), slot + k))
            slot += nseg
    return (np.asarray(it, np.int64).reshape(-1, 4), np.asarray(sp, np.int64).reshape(-1, 3))


def csc(n, indptr_local, src_local):
    """(ii): stable sort of CSR positions by source."""
    rows = len(indptr_local) - 1
    dst_local = np.repeat(np.arange(rows, dtype=np.int64), np.diff(indptr_local))
    cpos = np.argsort(np.asarray(src_local, np.int64), kind="stable")
    cindptr = np.zeros(n + 1, np.int64)
    cindptr[1:] = np.cumsum(np.bincount(np.asarray(src_local, np.int64), minlength=n))
    csr2csc = np.empty_like(cpos)
    csr2csc[cpos] = np.arange(len(cpos))
    return cindptr, dst_local[cpos], cpos, csr2csc


def build(indptr, indices, perm, num_parts=1, seg_edges=0):
    """The whole layout as a dict of numpy arrays (one entry per part)."""
    n = len(indptr) - 1
    new_of_old, ip, src, eid = relabel(indptr, indices, perm)
    m = int(ip[-1])
    S = seg_edges if seg_edges > 0 else auto_seg_edges(m)
    b = partition_bounds(ip, num_parts)
    parts = []
    for p in range(num_parts):
        r0, r1 = int(b[p]), int(b[p + 1])
        e0, e1 = int(ip[r0]), int(ip[r1])
        lip = ip[r0:r1 + 1] - e0
        lsrc = src[e0:e1]
        cip, cdst, cpos, c2 = csc(n, lip, lsrc)
        fi, fs = items(lip, S)
        bi, bs = items(cip, S)
        parts.append({"row_begin": r0, "row_end": r1, "indptr": lip, "src": lsrc, "eid": eid[e0:e1],
                      "cindptr": cip, "cdst": cdst, "cpos": cpos, "csr2csc": c2,
                      "fwd_items": fi, "fwd_splits": fs, "bwd_items": bi, "bwd_splits": bs})
    return {"perm": np.asarray(perm, np.int64), "new_of_old": new_of_old, "indptr": ip, "src": src,
            "eid": eid, "bounds": b, "seg_edges": S, "parts": parts}


def tile_unique_sources(indptr_new, src_new, tile_rows=64):
    """Sum over tiles of 64 consecutive rows of |unique sources| (the reuse
    statistic Σ|U_t|; E/Σ|U_t| is the average reuse of a staged source row)."""
    n = len(indptr_new) - 1
    tot = 0
    for t in range(0, n, tile_rows):
        a, b = int(indptr_new[t]), int(indptr_new[min(n, t + tile_rows)])
        tot += int(np.unique(src_new[a:b]).size)
    return tot
