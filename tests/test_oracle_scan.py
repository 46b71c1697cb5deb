"""Pins for the oracle's exclusive scan and binsearch_maxle (Figs. 4-5)."""
import numpy as np

import oracle
from golden_io import ints, load


def test_fig4_partition_map():
    g = load("fig4.txt")
    deg = ints(g["degrees"])
    ex = oracle.exclusive_scan(deg)
    assert list(ex[:-1]) == ints(g["exsum"])
    assert int(ex[-1]) == int(g["total"])
    want = [tuple(map(int, p.split(","))) for p in g["map"].split()]
    got = []
    for t in range(int(ex[-1])):
        i = oracle.maxle(ex[:-1], t)
        got.append((i, t - int(ex[i])))
    assert got == want


def test_fig5_block_byte_search():
    g = load("fig5.txt")
    pc = ints(g["popcounts"])
    ex = oracle.exclusive_scan(pc)
    assert list(ex[:-1]) == ints(g["exsum"])
    assert int(ex[-1]) == int(g["total"])
    assert [oracle.maxle(ex[:-1], t) for t in range(4)] == ints(g["target_byte"])


def test_maxle_ties_take_last():
    # reading C13: zero-degree entries (equal exsum values) are skipped
    a = np.array([0, 0, 3, 3, 3, 7], np.uint64)
    assert oracle.maxle(a, 0) == 1
    assert oracle.maxle(a, 2) == 1
    assert oracle.maxle(a, 3) == 4
    assert oracle.maxle(a, 100) == 5
    assert oracle.maxle(np.array([5], np.uint64), 4) == -1


def test_scan_matches_cumsum():
    rng = np.random.default_rng(0)
    a = rng.integers(0, 1 << 30, 1000).astype(np.uint64)
    ex = oracle.exclusive_scan(a)
    assert ex[0] == 0 and np.array_equal(ex[1:], np.cumsum(a, dtype=np.uint64))
    # maxle agrees with numpy's searchsorted(side='right') - 1 on the scan
    for t in rng.integers(0, int(ex[-1]), 50):
        assert oracle.maxle(ex[:-1], int(t)) == int(np.searchsorted(ex[:-1], t, "right") - 1)
