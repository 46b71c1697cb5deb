"""Pins for the oracle's Elias-Fano codec (oracle/oracle.c or_ef_*).

Independent anchors (none of them re-types the oracle's formulas):
  * Fig. 3 node 4 exact bytes (P:115 + footnote P:127, reading C6);
  * Fig. 2 stated numbers;
  * Fig. 6 forward-pointer numbers;
  * the paper's storage bound n(2 + ceil(log u/n)) bits and the
    information-theoretic facts that follow from the definition (upper-bits
    length = n stop bits + (u >> l) zeros);
  * exhaustive round trip over every sorted subset of [0, 12) and random lists,
    for several forward-pointer quanta k.
"""
import itertools
import math
from fractions import Fraction

import numpy as np
import pytest

import oracle
from golden_io import ints, load


def test_fig3_node4_exact_bytes():
    g = load("fig3_node4.txt")
    x = ints(g["list"])
    enc, l = oracle.ef_encode_list(x, k=512)
    assert l == int(g["l"])
    assert len(enc) == int(g["bytes"])
    assert enc.hex(" ") == g["hex"]
    assert oracle.ef_select1(enc, len(x), l, 512, 2) == int(g["select1_2"])
    assert list(oracle.ef_decode_list(enc, len(x), l, 512)) == x
    assert int(oracle.ef_decode_list(enc, len(x), l, 512)[2]) == int(g["x2"])


def test_fig2_stated_numbers():
    g = load("fig2.txt")
    x = ints(g["list"])
    n, u = int(g["n"]), int(g["u"])
    assert len(x) == n and x[-1] == u
    enc, l = oracle.ef_encode_list(x, k=0)
    assert l == int(g["l"])
    fb, lb, ub = oracle.ef_sections(n, u, 0)
    assert fb == 0
    # lower and upper halves are 16 bits each -> 2 bytes each, 4 bytes in total
    assert lb * 8 == int(g["lower_bits"])
    assert ub * 8 == int(g["upper_bits"])
    assert (lb + ub) * 8 == int(g["total_bits"])
    assert n * math.ceil(math.log2(u + 1)) == int(g["binary_bits"])
    assert oracle.ef_select1(enc, n, l, 0, 4) == int(g["select1_4"])
    dec = oracle.ef_decode_list(enc, n, l, 0)
    assert int(dec[4]) == int(g["x4"])
    assert (int(dec[7]) >> l) == int(g["upper_x7"])
    assert (int(dec[6]) >> l) == int(g["upper_x6"])
    # the gap of 3 between upper(x6) and upper(x7) is three 0s then the stop bit
    s6, s7 = oracle.ef_select1(enc, n, l, 0, 6), oracle.ef_select1(enc, n, l, 0, 7)
    assert s7 - s6 - 1 == int(g["upper_x7"]) - int(g["upper_x6"])


def test_fig6_forward_pointers():
    g = load("fig6.txt")
    x = ints(g["list"])
    k, a = int(g["k"]), int(g["a"])
    n = len(x)
    enc, l = oracle.ef_encode_list(x, k=k)
    assert (a + 1) // k - 1 == int(g["ptr_index_for_a"])
    assert n // k == 3
    assert oracle.ef_fwd(enc, 0) == int(g["fwd0"])
    assert oracle.ef_fwd(enc, 2) == int(g["fwd2"])
    assert oracle.ef_select1(enc, n, l, k, 7) == int(g["select1_7"])
    assert oracle.ef_select1(enc, n, l, k, 23) == int(g["select1_23"])
    # the pointers store select1(i) - i for i = k-1, 2k-1, ...
    for j in range(n // k):
        i = (j + 1) * k - 1
        assert oracle.ef_fwd(enc, j) == oracle.ef_select1(enc, n, l, k, i) - i
    assert list(oracle.ef_decode_list(enc, n, l, k)) == x


def _l_by_definition(n, u):
    """max{0, floor(log2(u/n))} by exact rational comparison."""
    if u < n:
        return 0
    q = Fraction(u, n)
    l = 0
    while Fraction(2 ** (l + 1)) <= q:
        l += 1
    return l


def test_lower_bits_definition():
    for n in range(1, 70):
        for u in list(range(0, 300)) + [2**31 - 1, 2**32 - 1, 3 * 2**20 + 5]:
            assert oracle.ef_lower_bits(n, u) == _l_by_definition(n, u), (n, u)


def _check_roundtrip(x, k):
    n = len(x)
    enc, l = oracle.ef_encode_list(x, k=k)
    u = x[-1]
    # size = 4*floor(n/k) + ceil(n*l/8) + ceil(((u>>l)+n)/8)  (C4, C7, C8)
    upper_bits = (u >> l) + n
    assert len(enc) == (4 * (n // k) if k else 0) + (n * l + 7) // 8 + (upper_bits + 7) // 8
    # north_star's a-priori size n*l + n + ceil(u / 2^l) bits: the upper
    # section's (u >> l) + n bits never exceed it, and equal it when 2^l | u
    # (reading C4: the last stop bit is the last bit, no trailing zero bucket)
    apriori = n * l + n + -(-u // (1 << l))
    assert n * l + upper_bits <= apriori <= n * l + upper_bits + 1
    assert (n * l + upper_bits == apriori) == (u % (1 << l) == 0)
    # at most n(2 + ceil(log u/n)) bits in total (u >= n case)
    if u >= n and u > 0:
        assert n * l + upper_bits <= n * (2 + math.ceil(math.log2(u / n))) + 1e-9
    # the upper-bits array holds exactly n ones, and the last one is its last bit
    # (it is the stop bit of x_{n-1}); decode reproduces the list
    dec = oracle.ef_decode_list(enc, n, l, k)
    assert list(map(int, dec)) == list(x)
    assert oracle.ef_select1(enc, n, l, k, n - 1) == upper_bits - 1
    for j in range(n // k if k else 0):
        i = (j + 1) * k - 1
        assert oracle.ef_fwd(enc, j) == (x[i] >> l)


def test_exhaustive_subsets_of_0_12():
    for mask in range(1, 1 << 12):
        x = [i for i in range(12) if mask >> i & 1]
        for k in (0, 1, 2, 3, 8):
            _check_roundtrip(x, k)


def test_random_lists_roundtrip():
    rng = np.random.default_rng(12345)
    for t in range(300):
        n = int(rng.integers(1, 3000))
        hi = int(rng.choice([n + 5, 4 * n, 1 << 20, 1 << 31, (1 << 32) - 1]))
        x = np.unique(rng.integers(0, hi, size=n, dtype=np.uint64)).astype(np.uint32)
        for k in (0, 512, int(rng.integers(1, 64))):
            _check_roundtrip([int(v) for v in x], k)


def test_nondecreasing_with_duplicates():
    # P:81 allows x_i <= x_{i+1}; the codec must handle equal values
    for x in ([0, 0, 0], [5, 5, 9, 9, 9, 100], [7] * 40):
        for k in (0, 4, 512):
            _check_roundtrip(x, k)


def test_complete_lists_l0():
    # lists of a complete graph: u < n -> l = 0, upper bits only
    for n in range(1, 40):
        x = list(range(n))
        enc, l = oracle.ef_encode_list(x, k=8)
        assert l == 0
        _check_roundtrip(x, 8)


@pytest.mark.parametrize("k", [0, 512])
def test_graph_level_offsets_are_exclusive_sums(k):
    # offsets = exclusive prefix sum of per-vertex compressed byte sizes
    rng = np.random.default_rng(7)
    n = 300
    src = rng.integers(0, n, 4000).astype(np.uint32)
    dst = rng.integers(0, n, 4000).astype(np.uint32)
    vlist, elist = oracle.csr_build(n, src, dst)
    offsets, nlb, data = oracle.efg_encode(vlist, elist, k)
    assert offsets[0] == 0 and int(offsets[-1]) == data.size
    for v in range(n):
        lst = elist[vlist[v]:vlist[v + 1]]
        enc, l = oracle.ef_encode_list(lst, k)
        assert int(offsets[v + 1] - offsets[v]) == len(enc)
        assert data[offsets[v]:offsets[v + 1]].tobytes() == enc
        assert nlb[v] == l
    dec = oracle.efg_decode_range(vlist, nlb, offsets, data, k, 0, n)
    assert np.array_equal(dec, elist)
