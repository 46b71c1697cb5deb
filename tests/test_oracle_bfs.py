"""Pins for the oracle's CSR construction and BFS depth (oracle/oracle.c).

Anchors: brute force over every simple graph on <= 5 vertices and random graphs
on <= 64 vertices (depth = hop distance computed by Floyd-Warshall in numpy, a
different algorithm from the oracle's FIFO queue); Python set-based adjacency for
the CSR (readings C11/C12); closed forms on path / star / complete /
disconnected graphs; Graph500-style invariants on an RMAT graph.
"""
import itertools

import numpy as np

import oracle
import synth


def _fw_dist(n, edges):
    INF = 10**9
    d = np.full((n, n), INF, np.int64)
    np.fill_diagonal(d, 0)
    for u, v in edges:
        if u != v:
            d[u, v] = 1
            d[v, u] = 1
    for k in range(n):
        d = np.minimum(d, d[:, [k]] + d[[k], :])
    d[d >= INF] = -1
    return d


def _csr_by_sets(n, src, dst, symmetrize=True):
    adj = [set() for _ in range(n)]
    for s, t in zip(src, dst):
        if s != t:
            adj[s].add(t)
            if symmetrize:
                adj[t].add(s)
    vlist = [0]
    elist = []
    for v in range(n):
        elist += sorted(adj[v])
        vlist.append(len(elist))
    return np.array(vlist, np.uint64), np.array(elist, np.uint32)


def test_csr_matches_set_construction():
    rng = np.random.default_rng(3)
    for t in range(50):
        n = int(rng.integers(1, 80))
        m = int(rng.integers(0, 400))
        src = rng.integers(0, n, m).astype(np.uint32)
        dst = rng.integers(0, n, m).astype(np.uint32)
        # duplicates and self loops on purpose
        if m:
            src[: m // 4] = dst[: m // 4]
        v1, e1 = oracle.csr_build(n, src, dst)
        v2, e2 = _csr_by_sets(n, src, dst)
        assert np.array_equal(v1, v2) and np.array_equal(e1, e2)


def test_csr_directed_keeps_orientation():
    src = np.array([0, 0, 2, 2, 2], np.uint32)
    dst = np.array([1, 1, 0, 2, 1], np.uint32)
    v, e = oracle.csr_build(3, src, dst, symmetrize=False)
    assert list(v) == [0, 1, 1, 3] and list(e) == [1, 0, 1]


def test_csr_rejects_out_of_range_ids():
    import pytest
    with pytest.raises(ValueError):
        oracle.csr_build(3, np.array([0, 3], np.uint32), np.array([1, 1], np.uint32))


def test_bfs_all_graphs_up_to_5_vertices():
    for n in range(1, 6):
        pairs = list(itertools.combinations(range(n), 2))
        for mask in range(1 << len(pairs)):
            edges = [pairs[i] for i in range(len(pairs)) if mask >> i & 1]
            src = np.array([e[0] for e in edges], np.uint32)
            dst = np.array([e[1] for e in edges], np.uint32)
            vlist, elist = oracle.csr_build(n, src, dst)
            d = _fw_dist(n, edges)
            for s in range(n):
                assert np.array_equal(oracle.bfs(vlist, elist, s), d[s]), (n, edges, s)


def test_bfs_random_graphs_up_to_64():
    rng = np.random.default_rng(11)
    for t in range(60):
        n = int(rng.integers(2, 65))
        m = int(rng.integers(0, 3 * n))
        src = rng.integers(0, n, m).astype(np.uint32)
        dst = rng.integers(0, n, m).astype(np.uint32)
        vlist, elist = oracle.csr_build(n, src, dst)
        d = _fw_dist(n, list(zip(src.tolist(), dst.tolist())))
        for s in rng.integers(0, n, 4):
            assert np.array_equal(oracle.bfs(vlist, elist, int(s)), d[int(s)])


def test_bfs_closed_forms():
    n = 50
    # path 0-1-...-49: depth = |index - s|
    src = np.arange(n - 1, dtype=np.uint32)
    dst = src + 1
    vlist, elist = oracle.csr_build(n, src, dst)
    for s in (0, 17, 49):
        assert np.array_equal(oracle.bfs(vlist, elist, s), np.abs(np.arange(n) - s))
    # star centred at 0
    src = np.zeros(n - 1, np.uint32)
    dst = np.arange(1, n, dtype=np.uint32)
    vlist, elist = oracle.csr_build(n, src, dst)
    d = oracle.bfs(vlist, elist, 5)
    assert d[5] == 0 and d[0] == 1 and all(d[v] == 2 for v in range(1, n) if v != 5)
    # complete graph K_12
    pairs = list(itertools.combinations(range(12), 2))
    vlist, elist = oracle.csr_build(12, np.array([p[0] for p in pairs], np.uint32),
                                    np.array([p[1] for p in pairs], np.uint32))
    assert list(oracle.bfs(vlist, elist, 3)) == [1] * 3 + [0] + [1] * 8
    # isolated source and a self-loop-only vertex
    vlist, elist = oracle.csr_build(4, np.array([1, 3], np.uint32), np.array([2, 3], np.uint32))
    assert list(oracle.bfs(vlist, elist, 0)) == [0, -1, -1, -1]
    assert list(oracle.bfs(vlist, elist, 3)) == [-1, -1, -1, 0]


def graph500_validate(vlist, elist, source, depth):
    """Graph500-style invariants; together they characterise the hop distance."""
    n = vlist.size - 1
    deg = np.diff(vlist).astype(np.int64)
    u = np.repeat(np.arange(n), deg)
    v = elist.astype(np.int64)
    du, dv = depth[u], depth[v]
    assert depth[source] == 0
    both = (du >= 0) & (dv >= 0)
    assert np.all(np.abs(du[both] - dv[both]) <= 1)
    assert not np.any((du >= 0) != (dv >= 0))
    # every reached v != source has a neighbour at depth-1
    has_parent = np.zeros(n, bool)
    ok = both & (du == dv - 1)
    has_parent[v[ok]] = True
    reached = depth >= 0
    reached[source] = False
    assert np.all(has_parent[reached])


def test_bfs_rmat_invariants():
    n, src, dst = synth.rmat(12, 16, seed=1)
    vlist, elist = oracle.csr_build(n, src, dst)
    for s in (0, 1, 100):
        graph500_validate(vlist, elist, s, oracle.bfs(vlist, elist, s))


def test_bfs_bounded_sample():
    """or_bfs_bounded (bench.py reference-arm sample): every depth it assigns is
    the Floyd-Warshall hop distance, it scans at least the budget (or finishes
    the BFS), the scanned count is the degree sum of the dequeued vertices, and
    an unlimited budget is the full BFS."""
    rng = np.random.default_rng(12)
    for t in range(40):
        n = int(rng.integers(2, 65))
        m = int(rng.integers(0, 4 * n))
        src = rng.integers(0, n, m).astype(np.uint32)
        dst = rng.integers(0, n, m).astype(np.uint32)
        vlist, elist = oracle.csr_build(n, src, dst)
        deg = np.diff(vlist)
        d = _fw_dist(n, list(zip(src.tolist(), dst.tolist())))
        for s in rng.integers(0, n, 3):
            s = int(s)
            full = d[s]
            for budget in (0, 1, 5, int(rng.integers(0, 2 * m + 2)), 2**63):
                got, nv, scanned = oracle.bfs_bounded(vlist, elist, s, budget)
                assigned = got >= 0
                assert np.array_equal(got[assigned], full[assigned])
                assert got[s] == 0
                # the dequeued vertices are the nv closest (FIFO order: by depth)
                reached = int((full >= 0).sum())
                assert nv <= reached
                assert scanned >= min(budget, int(deg[full >= 0].sum())) or nv == reached
                if budget == 2**63:
                    assert np.array_equal(got, full) and nv == reached
                    assert scanned == int(deg[full >= 0].sum())
                # every vertex at depth < the last dequeued depth was dequeued, hence
                # all of its neighbours have depths assigned
                if nv:
                    dq_depths = np.sort(full[full >= 0])[:nv]
                    for u in np.flatnonzero((full >= 0) & (full < dq_depths[-1])):
                        assert np.all(got[elist[vlist[u]:vlist[u + 1]]] >= 0)


def test_cpu_baseline_omp_bfs_matches_oracle():
    """The optional all-core CPU baseline (cpu_baseline/omp_bfs.c) gives the
    oracle's depths (a reported baseline must compute the same thing)."""
    import cpu_baseline
    n, src, dst = synth.rmat(14, 16, seed=9)
    vlist, elist = oracle.csr_build(n, src, dst)
    for s in (0, 1, 5000, n - 1):
        ref = oracle.bfs(vlist, elist, s)
        for t in (1, 4):
            assert np.array_equal(cpu_baseline.bfs(vlist, elist, s, threads=t), ref)
