"""NEXT-2 product layout (csrc/band.cpp through the C ABI) against the band oracle
(oracle/band.py): the path P, the coverage owners and the directed multiplicities
must match bit-exactly (SURVEY §8(c) "layout must match the oracle bit-exactly");
partial slots group each multi-appearance node's appearances in order.  CPU only
(host build; no compute call)."""
import numpy as np
import pytest

from oracle import band as ob
from paper_conf_icdcs_dengr24_b200 import mega as M
from synth import random_multigraph


def oracle_masks(n, ip, ix, window):
    tr = ob.traverse_faithful(n, ip, ix, window=window)
    band = ob.band_layout(n, ip, ix, tr)
    P = band["P"]
    L = len(P)
    own = np.zeros(L, np.uint64)
    for t, offs in enumerate(tr["owner"]):
        for o in offs:
            own[t] |= np.uint64(1 << (o - 1))
    lm, rm = np.zeros(L, np.uint64), np.zeros(L, np.uint64)
    lc, rc = {}, {}
    for t, o, cf, cb in band["pairs"]:
        if cf:
            lm[t] |= np.uint64(1 << (o - 1))
            lc[(t, o)] = cf
        if cb:
            rm[t - o] |= np.uint64(1 << (o - 1))
            rc[(t - o, o)] = cb
    cnt = []
    first = set()
    for t in range(L):
        for o in range(1, window + 1):
            if (int(lm[t]) >> (o - 1)) & 1:
                cnt.append(lc[(t, o)])
        for o in range(1, window + 1):
            if (int(rm[t]) >> (o - 1)) & 1:
                cnt.append(rc[(t, o)])
        x = int(P[t])
        if x not in first:
            first.add(x)
            if band["self_loops"][x]:
                cnt.append(int(band["self_loops"][x]))
    return tr, P, own, lm, rm, np.asarray(cnt, np.uint16)


@pytest.mark.parametrize("seed", range(10))
@pytest.mark.parametrize("window", [1, 2, 5])
def test_band_bit_exact(seed, window):
    ip, ix = random_multigraph(300 + seed, 45, 200, undirected=seed % 2 == 0, isolated=3)
    n = len(ip) - 1
    tr, P, own, lm, rm, cnt = oracle_masks(n, ip, ix, window)
    v = M.mega_band_build(ip, ix, window=window).view()
    assert np.array_equal(v["P"], P)
    assert np.array_equal(v["own"], own)
    assert np.array_equal(v["lmask"], lm) and np.array_equal(v["rmask"], rm)
    assert np.array_equal(v["cnt"], cnt)
    assert v["jumps"] == tr["jumps"] and v["virtual_edges"] == tr["virtual"]
    # partial slots: nodes with > 1 appearance, their appearances in order, consecutive slots
    napp = np.bincount(P, minlength=n)
    for node, s0, ns in v["merges"]:
        assert napp[node] == ns > 1
        ts = np.nonzero(P == node)[0]
        assert v["slot"][ts].tolist() == list(range(s0, s0 + ns))
    assert np.all(v["slot"][napp[P] == 1] == -1)


def test_band_errors():
    ip = np.array([0, 1], np.int64)
    ix = np.array([0], np.int32)
    with pytest.raises(M.MegaError):
        M.mega_band_build(ip, ix, window=65)
