"""Host logic of the k-GPU forward split (CPU; SURVEY §8(e) forward steps 2-4).

mega_preprocess's parts are read through mega_layout_dist_view_get: per part,
the items of the local pass (in-edges whose source the part owns: block (p,p),
computable before the exchange lands), the items of the remote pass, and the
merge records of rows whose edges end up in several items.  Checked here:
  * every in-edge of the part is in exactly one item, local items only reference
    the part's own sources and remote items never do;
  * slots form one contiguous block per merged row, single-item rows are
    finalised in place (slot -1), rows without in-edges by the local pass;
  * the backward's own-source ranges hold exactly the own sources;
  * fp64 arithmetic over the items (partial softmax states per item, then the
    fixed-order merge M = max m_k, L = sum l_k e^(m_k - M), out = sum acc_k
    e^(m_k - M) / L) reproduces the oracle's forward on every row of the part.
"""
import numpy as np
import pytest

import synth
from oracle import gat as og
from paper_conf_icdcs_dengr24_b200 import mega as M


def _graphs():
    yield "multigraph", synth.random_multigraph(31, 400, 5000, undirected=False, isolated=12), 16
    cfg = synth.scaled(synth.CONFIGS["reddit"], 1500, 40000)
    ip, ix, _ = synth.make_graph(cfg)
    yield "reddit-scaled", (ip, ix), 64


@pytest.mark.parametrize("k", [2, 3, 5])
def test_dist_items_partition_and_merge(k):
    rng = np.random.default_rng(k)
    for name, (ip, ix), seg in _graphs():
        n = len(ip) - 1
        H, F = 2, 4
        Wh_old = rng.standard_normal((n, H, F))
        a_l, a_r = rng.standard_normal((H, F)), rng.standard_normal((H, F))
        lay = M.mega_preprocess(ip, ix, num_parts=k, seg_edges=seg)
        v0 = lay.view(0)
        perm = v0["perm"].astype(np.int64)
        bounds = v0["bounds"]
        Wh = Wh_old[perm]
        # oracle forward on the whole graph, in new ids
        ip_new = np.zeros(n + 1, np.int64)
        srcs = []
        for p in range(k):
            v = lay.view(p)
            ip_new[v["row_begin"] + 1:v["row_end"] + 1] = v["indptr"][1:] + ip_new[v["row_begin"]]
            srcs.append(v["src"])
        ref = og.gat_forward(ip_new, np.concatenate(srcs), Wh, a_l, a_r)
        el, er = og.attention_halves(Wh, a_l, a_r)
        for p in range(k):
            v = lay.view(p)
            d = M.mega_layout_dist_view_get(lay, p)
            b0, b1 = int(bounds[p]), int(bounds[p + 1])
            E = int(v["part_edges"])
            src = v["src"].astype(np.int64)
            cover = np.zeros(E, np.int64)
            for items, local in ((d["local_items"], True), (d["remote_items"], False)):
                for r, e0, e1, slot in items:
                    cover[e0:e1] += 1
                    own = (src[e0:e1] >= b0) & (src[e0:e1] < b1)
                    assert own.all() if local else not own.any(), (name, p, r, local)
                    assert v["indptr"][r] <= e0 <= e1 <= v["indptr"][r + 1]
            assert np.all(cover == 1), (name, p)
            # slots and merge records
            allit = np.concatenate([d["local_items"], d["remote_items"]])
            slotted = allit[allit[:, 3] >= 0]
            assert len(np.unique(slotted[:, 3])) == len(slotted) == d["num_slots"]
            for r, s0, ns in d["splits"]:
                mine = slotted[(slotted[:, 3] >= s0) & (slotted[:, 3] < s0 + ns)]
                assert len(mine) == ns >= 2 and np.all(mine[:, 0] == r)
            rows_with_items = np.concatenate([allit[:, 0]])
            assert set(rows_with_items.tolist()) == set(range(b1 - b0))
            deg = np.diff(v["indptr"])
            for r in np.flatnonzero(deg == 0):
                assert [r, v["indptr"][r], v["indptr"][r], -1] in d["local_items"].tolist()
            # backward own-source ranges (bwd_items are (source, ...) sorted by source)
            bi = v["bwd_items"]
            i0, i1 = d["bwd_own_items_begin"], d["bwd_own_items_end"]
            assert np.all((bi[i0:i1, 0] >= b0) & (bi[i0:i1, 0] < b1))
            assert not np.any((bi[:i0, 0] >= b0) & (bi[:i0, 0] < b1))
            assert not np.any((bi[i1:, 0] >= b0) & (bi[i1:, 0] < b1))
            # fp64 arithmetic over the items, then the merge
            state = {}
            out = np.zeros((b1 - b0, H, F))
            lse = np.full((b1 - b0, H), -np.inf)
            for r, e0, e1, slot in allit:
                g = b0 + r
                z = el[g][None] + er[src[e0:e1]]
                s = np.where(z > 0, z, og.SLOPE * z)
                m = s.max(0) if e1 > e0 else np.full(H, -np.inf)
                pexp = np.exp(s - m) if e1 > e0 else np.zeros((0, H))
                l_ = pexp.sum(0)
                acc = np.einsum("eh,ehf->hf", pexp, Wh[src[e0:e1]]) if e1 > e0 else np.zeros((H, F))
                if slot < 0:
                    if e1 > e0:
                        out[r] = acc / l_[:, None]
                        lse[r] = m + np.log(l_)
                else:
                    state[slot] = (m, l_, acc)
            for r, s0, ns in d["splits"]:
                ms = np.stack([state[s][0] for s in range(s0, s0 + ns)])
                Mx = ms.max(0)
                f = np.exp(ms - Mx)
                L = sum(state[s][1] * f[i] for i, s in enumerate(range(s0, s0 + ns)))
                A = sum(state[s][2] * f[i][:, None] for i, s in enumerate(range(s0, s0 + ns)))
                out[r] = A / L[:, None]
                lse[r] = Mx + np.log(L)
            assert np.allclose(out, ref["out"][b0:b1], rtol=1e-12, atol=1e-12), (name, p)
            assert np.array_equal(np.isinf(lse), np.isinf(ref["lse"][b0:b1]))
            fin = np.isfinite(lse)
            assert np.allclose(lse[fin], ref["lse"][b0:b1][fin], rtol=1e-12, atol=1e-12)


def test_single_part_has_no_dist_items():
    ip, ix = synth.random_multigraph(2, 50, 300)
    d = M.mega_layout_dist_view_get(M.mega_preprocess(ip, ix), 0)
    assert d["num_local_items"] == d["num_remote_items"] == d["num_splits"] == 0


@pytest.mark.parametrize("k", [2, 4])
def test_halo_plan(k):
    """NEXT-1: part p receives from q exactly the rows of q its edges reference, and the
    list p sends to q is the list q receives from p (same order: the packed buffers line up)."""
    cfg = synth.scaled(synth.CONFIGS["products"], 4000, 60000)
    ip, ix, _ = synth.make_graph(cfg)
    lay = M.mega_preprocess(ip, ix, num_parts=k)
    b = lay.view(0)["bounds"]
    views = [lay.view(p) for p in range(k)]
    dv = [M.mega_layout_dist_view_get(lay, p) for p in range(k)]
    for p in range(k):
        ref = np.unique(views[p]["src"])
        for q in range(k):
            r = dv[p]["recv_idx"][dv[p]["recv_off"][q]:dv[p]["recv_off"][q + 1]]
            if q == p:
                assert len(r) == 0
                continue
            assert np.array_equal(r, ref[(ref >= b[q]) & (ref < b[q + 1])])
            s_qp = dv[q]["send_idx"][dv[q]["send_off"][p]:dv[q]["send_off"][p + 1]]
            assert np.array_equal(s_qp, r)
        assert dv[p]["num_recv"] == dv[p]["recv_off"][-1] <= dv[p]["full_recv_rows"]
        assert dv[p]["full_recv_rows"] == cfg.n - (b[p + 1] - b[p])
