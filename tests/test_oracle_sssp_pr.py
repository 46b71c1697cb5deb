"""Pins for the oracle's SSSP (fp32 Dijkstra) and PageRank (fp64), §VI-F.

SSSP anchors: scipy's fp64 Dijkstra on the same graph (agreement within fp32
rounding of the path sums), a Bellman-Ford fixpoint computed in fp32 numpy with
a different relaxation order (bit-exact: DESIGN.md reading C20 argues the fp32
fixpoint is unique), closed forms on a path.
PageRank anchors: the d-regular closed form (uniform 1/N), a dense numpy matrix
power iteration (a different formulation), and the star graph's stationary
ratio.
"""
import itertools

import numpy as np
import scipy.sparse as sp
from scipy.sparse.csgraph import dijkstra

import oracle
import synth


def _graph(n, m, seed):
    rng = np.random.default_rng(seed)
    src = rng.integers(0, n, m).astype(np.uint32)
    dst = rng.integers(0, n, m).astype(np.uint32)
    vlist, elist = oracle.csr_build(n, src, dst)
    u = np.repeat(np.arange(n, dtype=np.uint32), np.diff(vlist).astype(np.int64))
    w = np.array([synth.weight_pair(2000 + seed, int(a), int(b)) for a, b in zip(u, elist)],
                 np.float32)
    return vlist, elist, u, w


def test_sssp_vs_scipy_fp64():
    for seed in range(10):
        n = 60
        vlist, elist, u, w = _graph(n, 200, seed)
        A = sp.csr_matrix((w.astype(np.float64), elist, vlist.astype(np.int64)), shape=(n, n))
        ref = dijkstra(A, directed=True, indices=0)
        got = oracle.sssp(vlist, elist, w, 0)
        fin = np.isfinite(ref)
        assert np.array_equal(fin, np.isfinite(got))
        assert np.allclose(got[fin], ref[fin], rtol=1e-6, atol=0)


def _bellman_ford_fp32(n, vlist, elist, u, w, s):
    d = np.full(n, np.inf, np.float32)
    d[s] = 0
    while True:
        cand = (d[u] + w).astype(np.float32)
        nd = d.copy()
        np.minimum.at(nd, elist, cand)
        if np.array_equal(nd, d):
            return d
        d = nd


def test_sssp_fp32_fixpoint_bit_exact():
    for seed in range(20):
        n = 50
        vlist, elist, u, w = _graph(n, 180, 100 + seed)
        got = oracle.sssp(vlist, elist, w, 3)
        ref = _bellman_ford_fp32(n, vlist, elist, u, w, 3)
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


def test_sssp_path_closed_form():
    n = 20
    src = np.arange(n - 1, dtype=np.uint32)
    dst = src + 1
    vlist, elist = oracle.csr_build(n, src, dst)
    w = np.full(elist.size, 0.25, np.float32)
    d = oracle.sssp(vlist, elist, w, 0)
    assert np.array_equal(d, 0.25 * np.arange(n, dtype=np.float32))


def test_pagerank_regular_graph_uniform():
    # cycle C_n and K_n are regular -> PR = 1/N at every iteration
    for n in (5, 17):
        src = np.arange(n, dtype=np.uint32)
        dst = (src + 1) % n
        vlist, elist = oracle.csr_build(n, src, dst)
        assert np.allclose(oracle.pagerank(vlist, elist), 1.0 / n, rtol=1e-14)
    pairs = list(itertools.combinations(range(9), 2))
    vlist, elist = oracle.csr_build(9, np.array([p[0] for p in pairs], np.uint32),
                                    np.array([p[1] for p in pairs], np.uint32))
    assert np.allclose(oracle.pagerank(vlist, elist), 1.0 / 9, rtol=1e-14)


def test_pagerank_dense_power_iteration():
    rng = np.random.default_rng(5)
    for t in range(10):
        n = int(rng.integers(3, 40))
        m = int(rng.integers(0, 3 * n))
        src = rng.integers(0, n, m).astype(np.uint32)
        dst = rng.integers(0, n, m).astype(np.uint32)
        vlist, elist = oracle.csr_build(n, src, dst)
        A = np.zeros((n, n))
        for v in range(n):
            for x in elist[vlist[v]:vlist[v + 1]]:
                A[x, v] = 1.0
        deg = A.sum(axis=0)
        # column-stochastic transition with dangling columns -> uniform
        M = np.where(deg > 0, A / np.where(deg > 0, deg, 1), 1.0 / n)
        r = np.full(n, 1.0 / n)
        for _ in range(50):
            r = (1 - 0.85) / n + 0.85 * (M @ r)
        got = oracle.pagerank(vlist, elist, 0.85, 50)
        assert np.allclose(got, r, rtol=1e-12, atol=1e-15)
        assert abs(got.sum() - 1.0) < 1e-12


def test_pagerank_star_ratio():
    # star K_{1,s}: stationary ratio centre/leaf solves the 2-state chain
    s = 10
    src = np.zeros(s, np.uint32)
    dst = np.arange(1, s + 1, dtype=np.uint32)
    vlist, elist = oracle.csr_build(s + 1, src, dst)
    r = oracle.pagerank(vlist, elist, 0.85, 200)
    N = s + 1
    d = 0.85
    # centre c and leaf l: c = (1-d)/N + d*s*l ; l = (1-d)/N + d*c/s — the 2x2 linear system
    Amat = np.array([[1.0, -d * s], [-d / s, 1.0]])
    b = np.array([(1 - d) / N, (1 - d) / N])
    c_ref, l_ref = np.linalg.solve(Amat, b)
    assert np.allclose(r[0], c_ref, rtol=1e-12)
    assert np.allclose(r[1:], l_ref, rtol=1e-12)
