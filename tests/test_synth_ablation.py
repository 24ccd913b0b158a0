"""The community-sorted ablation order (bench.py --order community) uses
the generator's own community assignment and a pure relabelling of the graph.  CPU only."""
import numpy as np

import synth


def test_communities_match_the_generator_draws():
    cfg = synth.scaled(synth.CONFIGS["products"], 3000, 40000)
    c = synth.communities(cfg)
    lib = synth._load()
    seed = (cfg.seed ^ 0x2222222222222222) & 0xFFFFFFFFFFFFFFFF
    assert [int(x) for x in c[:200]] == [lib.msynth_draw(seed, v) % cfg.communities for v in range(200)]
    ip, ix, _ = synth.make_graph(cfg)
    dst = np.repeat(np.arange(cfg.n), np.diff(ip))
    assert abs(np.mean(c[dst] == c[ix]) - cfg.mu) < 0.03      # the generator's homophily


def test_relabel_preserves_the_edge_multiset():
    ip, ix = synth.random_multigraph(5, 200, 3000, undirected=False, isolated=7)
    n = len(ip) - 1
    order = np.random.default_rng(1).permutation(n)
    ip2, ix2 = synth.relabel(ip, ix, order)
    old = sorted(zip(np.repeat(np.arange(n), np.diff(ip)).tolist(), ix.tolist()))
    new = sorted(zip(order[np.repeat(np.arange(n), np.diff(ip2))].tolist(), order[ix2].tolist()))
    assert old == new
