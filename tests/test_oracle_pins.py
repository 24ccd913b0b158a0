"""Pins for the oracle's ablation orders and the reuse statistic (SURVEY §8(c)-c2(v),
§8(d)-d3), from values fixed outside the oracle: hand counts and the published
SplitMix64 test vector.  CPU only.

The ablation orders replace traversal R in mega_preprocess (MEGA_ORDER_DEGREE,
MEGA_ORDER_RANDOM; include/mega.h); test_layout_product.py then checks the
product against these oracle functions, so a wrong draw index or tie-break in
the oracle would otherwise go unnoticed.
"""
import numpy as np

from oracle import layout as ol
from oracle import traverse as ot

# SplitMix64 (Steele, Lea, Flood 2014; the reference generator of Vigna's
# xoshiro page): state 0, first three outputs.  Published constants, not
# computed by the oracle.
SPLITMIX64_SEED0 = (0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F)


def test_order_random_follows_published_splitmix_draws():
    # Fisher-Yates over [0, 1, 2, 3] with seed 0: step i = 3, 2, 1
    # takes the next SplitMix64 output u and swaps p[i] with p[(u >> 11) % (i + 1)].
    #   i = 3: (0xE220A8397B1DCDAF >> 11) % 4 = 1 -> [0, 3, 2, 1]
    #   i = 2: (0x6E789E6AA1B965F4 >> 11) % 3 = 0 -> [2, 3, 0, 1]
    #   i = 1: (0x06C45D188009454F >> 11) % 2 = 0 -> [3, 2, 0, 1]
    assert [(u >> 11) % m for u, m in zip(SPLITMIX64_SEED0, (4, 3, 2))] == [1, 0, 0]
    assert ot.order_random(4, 0).tolist() == [3, 2, 0, 1]
    # n = 1 draws nothing; every order is a permutation
    assert ot.order_random(1, 7).tolist() == [0]
    for n, seed in ((10, 1), (257, 99)):
        assert sorted(ot.order_random(n, seed).tolist()) == list(range(n))


def test_order_degree_hand_counted():
    # in-degrees [1, 3, 0, 3, 2] -> stable sort by (-in-degree, id): 1, 3 (deg 3; id tie), 4, 0, 2
    indptr = np.array([0, 1, 4, 4, 7, 9])
    assert ot.order_degree(5, indptr).tolist() == [1, 3, 4, 0, 2]
    # all equal degrees keep the identity order
    assert ot.order_degree(4, np.array([0, 2, 4, 6, 8])).tolist() == [0, 1, 2, 3]


def test_tile_unique_sources_hand_counted():
    # rows (new ids) and their sources; tiles of 2 rows:
    #   tile {0, 1}: sources {0, 1} and {1, 1}  -> {0, 1}     = 2
    #   tile {2, 3}: sources {2, 2} and {}      -> {2}        = 1
    #   tile {4}:    sources {0, 3, 4}          -> {0, 3, 4}  = 3
    indptr = np.array([0, 2, 4, 6, 6, 9])
    src = np.array([0, 1, 1, 1, 2, 2, 0, 3, 4])
    assert ol.tile_unique_sources(indptr, src, tile_rows=2) == 2 + 1 + 3
    # one tile over everything = number of distinct sources; tile of 1 row = sum of per-row distinct counts
    assert ol.tile_unique_sources(indptr, src, tile_rows=64) == 5
    assert ol.tile_unique_sources(indptr, src, tile_rows=1) == 2 + 1 + 1 + 0 + 3
