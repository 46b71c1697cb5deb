"""GPU parity tests: the CUDA path (through the C ABI) vs the CPU oracle.

Bit-exact comparisons (integer work):
  * efg_decode of every neighbour list == the oracle's CSR elist
    (steps a1-a5: frontier/record gather, scan, tile partition, chunk bit
    ranges via forward pointers, EF element decode);
  * efg_bfs depth == oracle FIFO-BFS depth (steps a1-a7);
  * parents are checked by invariant (several valid answers).
Sizes span many edge tiles (2048 edges) and chunk boundaries (k), with ragged
tails; special graphs cover the degenerate cases.
"""
import itertools

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def efg(cuda_ok):
    import paper_conf_ipps_gerak23_b200 as m
    return m


def _check_decode(efg, n, src, dst, k, **kw):
    g = efg.Graph.build(n, src, dst, k=k, **kw)
    ov, oe = oracle.csr_build(n, src, dst, **({} if "flags" not in kw else
                                               {"symmetrize": bool(kw["flags"] & 1)}))
    got = g.decode(0, n)
    assert got.size == oe.size
    assert np.array_equal(got, oe)
    return g, ov, oe


def _check_bfs(g, ov, oe, sources):
    for s in sources:
        d = g.bfs(int(s))
        ref = oracle.bfs(ov, oe, int(s))
        assert np.array_equal(d, ref), f"source {s}: {np.flatnonzero(d != ref)[:10]}"


@pytest.mark.parametrize("k", [512, 64, 8, 0])
def test_decode_and_bfs_rmat(efg, k):
    n, src, dst = synth.rmat(14, 16, seed=1)
    g, ov, oe = _check_decode(efg, n, src, dst, k)
    _check_bfs(g, ov, oe, [0, 1, 2, 12345, n - 1])
    g.free()


def test_c1_rmat16_100_sources(efg):
    # BASELINE.json configs[0]: RMAT scale 16, edgefactor 16, BFS from vertex 0
    n, src, dst = synth.config_edges(1)
    g, ov, oe = _check_decode(efg, n, src, dst, 512)
    deg = np.diff(ov)
    srcs = synth.sources(n, 100, seed=1001, nonisolated_mask=deg > 0)
    _check_bfs(g, ov, oe, np.concatenate([[0], srcs]))
    g.free()


def test_decode_partial_ranges(efg):
    n, src, dst = synth.rmat(12, 16, seed=3)
    g = efg.Graph.build(n, src, dst, k=16)
    ov, oe = oracle.csr_build(n, src, dst)
    rng = np.random.default_rng(0)
    for _ in range(20):
        a, b = sorted(rng.integers(0, n + 1, 2))
        got = g.decode(int(a), int(b))
        assert np.array_equal(got, oe[ov[a]:ov[b]])
    g.free()


def test_decode_to_device_buffer(efg):
    import torch
    n, src, dst = synth.rmat(12, 8, seed=4)
    g = efg.Graph.build(n, src, dst)
    ov, oe = oracle.csr_build(n, src, dst)
    out = torch.empty(oe.size, dtype=torch.int32, device="cuda")
    g.decode(0, n, out)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy().view(np.uint32), oe)
    # depth into a device buffer
    d = torch.empty(n, dtype=torch.int32, device="cuda")
    g.bfs(0, depth=d)
    torch.cuda.synchronize()
    assert np.array_equal(d.cpu().numpy(), oracle.bfs(ov, oe, 0))
    g.free()


def test_long_lists_cross_forward_pointers(efg):
    # hubs with degrees around 1x, 2x, 3x k and many small lists; wide ids
    rng = np.random.default_rng(9)
    n = 200_000
    srcs, dsts = [], []
    for hub, deg in [(0, 511), (1, 512), (2, 513), (3, 1024), (4, 1537), (n - 1, 5000), (7, 70000)]:
        nb = rng.choice(n, size=deg, replace=False).astype(np.uint32)
        srcs.append(np.full(deg, hub, np.uint32))
        dsts.append(nb)
    srcs.append(rng.integers(0, n, 300000).astype(np.uint32))
    dsts.append(rng.integers(0, n, 300000).astype(np.uint32))
    src, dst = np.concatenate(srcs), np.concatenate(dsts)
    for k in (512, 32):
        g, ov, oe = _check_decode(efg, n, src, dst, k)
        _check_bfs(g, ov, oe, [0, 7, n - 1, 12345])
        g.free()


def test_dense_lists_l0(efg):
    # complete graph: every list has u < n -> l = 0; also two cliques, disconnected
    pairs = list(itertools.combinations(range(300), 2))
    src = np.array([p[0] for p in pairs], np.uint32)
    dst = np.array([p[1] for p in pairs], np.uint32)
    src = np.concatenate([src, src + 400])
    dst = np.concatenate([dst, dst + 400])
    n = 800
    g, ov, oe = _check_decode(efg, n, src, dst, 512)
    _check_bfs(g, ov, oe, [0, 299, 400, 350, 799])
    g.free()


def test_special_graphs(efg):
    # path (depth = index), star, isolated source, self-loop-only vertex
    n = 10000
    src = np.arange(n - 1, dtype=np.uint32)
    g, ov, oe = _check_decode(efg, n, src, src + 1, 512)
    d = g.bfs(0)
    assert np.array_equal(d, np.arange(n))
    g.free()
    src = np.zeros(n - 1, np.uint32)
    g, ov, oe = _check_decode(efg, n, src, np.arange(1, n, dtype=np.uint32), 512)
    _check_bfs(g, ov, oe, [0, 5, n - 1])
    g.free()
    g = efg.Graph.build(5, np.array([1, 4], np.uint32), np.array([2, 4], np.uint32))
    assert list(g.bfs(0)) == [0, -1, -1, -1, -1]
    assert list(g.bfs(4)) == [-1, -1, -1, -1, 0]
    assert list(g.bfs(2)) == [-1, 1, 0, -1, -1]
    g.free()


def test_directed_graph(efg):
    n, src, dst = synth.rmat(12, 8, seed=5)
    g = efg.Graph.build(n, src, dst, flags=efg.EFG_DEDUP | efg.EFG_DROP_SELF_LOOPS)
    ov, oe = oracle.csr_build(n, src, dst, symmetrize=False)
    assert np.array_equal(g.decode(0, n), oe)
    _check_bfs(g, ov, oe, [0, 1, 100])
    g.free()


def test_directed_sink_below_visited_prefix(efg):
    """A directed sink (out-degree 0, but an in-edge) with a smaller id than
    every unvisited non-sink vertex must still be probed: the visited prefix
    counts only vertices without in-edges as never probed."""
    flags = efg.EFG_DEDUP | efg.EFG_DROP_SELF_LOOPS
    src = np.array([1, 1, 2], np.uint32)
    dst = np.array([0, 2, 1], np.uint32)
    g = efg.Graph.build(3, src, dst, flags=flags)
    ov, oe = oracle.csr_build(3, src, dst, symmetrize=False)
    _check_bfs(g, ov, oe, [1, 2])
    g.free()
    # many sinks at the low ids, sources among the high ids
    rng = np.random.default_rng(7)
    n = 4096
    s = rng.integers(n // 2, n, 40000).astype(np.uint32)
    d = rng.integers(0, n, 40000).astype(np.uint32)
    g = efg.Graph.build(n, s, d, flags=flags)
    ov, oe = oracle.csr_build(n, s, d, symmetrize=False)
    _check_bfs(g, ov, oe, [n // 2, n - 1, 3000])
    g.free()


@pytest.mark.parametrize("reorder", [False, True])
def test_prefix_skip_on_off_identical(efg, reorder):
    """EFG_OPT_PREFIX_SKIP only drops work on ids below the visited prefix:
    depths with and without it equal the oracle's."""
    n, src, dst = synth.rmat(14, 16, seed=11)
    flags = efg.EFG_DEFAULT_FLAGS | (efg.EFG_REORDER_DEGREE if reorder else 0)
    g = efg.Graph.build(n, src, dst, flags=flags)
    ov, oe = oracle.csr_build(n, src, dst)
    deg = np.diff(ov)
    srcs = synth.sources(n, 6, 77, deg > 0)
    for on in (False, True, False):
        g.set_prefix_skip(on)
        _check_bfs(g, ov, oe, srcs)
        g.set_level_loop(True)
        _check_bfs(g, ov, oe, srcs[:2])
        g.set_level_loop(False)
    g.free()


@pytest.mark.parametrize("k", [512, 32])
def test_expand_variants_identical(efg, k):
    """Every EFG_OPT_EXPAND_VARIANT mask (decode paths, staging, frontier order,
    work assignment, level-end list skip) only changes how
    the work is done: BFS depths equal the oracle's, decoded lists its CSR, SSSP
    distances the fp32 Dijkstra — on a degree-relabelled RMAT graph (skewed
    batches: both decode paths) and an unrelabelled one."""
    n, src, dst = synth.rmat(15, 16, seed=5)
    w = synth.weights(src, dst, seed=2005)
    ov, oe = oracle.csr_build(n, src, dst)
    deg = np.diff(ov)
    srcs = synth.sources(n, 3, 555, deg > 0)
    for reorder in (True, False):
        flags = efg.EFG_DEFAULT_FLAGS | (efg.EFG_REORDER_DEGREE if reorder else 0)
        g = efg.Graph.build(n, src, dst, k=k, flags=flags, weights=w)
        u = np.repeat(np.arange(n, dtype=np.uint32), deg.astype(np.int64))
        dref = oracle.sssp(ov, oe, synth.weights(u, oe, seed=2005), int(srcs[0]))
        for mask in (0, 1, 2, 3, 4, 8, 11, 16, 27, 32, 43, 59, 63, 107, 127):
            g.set_expand_variant(mask)
            _check_bfs(g, ov, oe, srcs)
            g.set_level_loop(True)
            _check_bfs(g, ov, oe, srcs[:1])
            g.set_level_loop(False)
            if mask in (0, 11, 43, 63):
                if not reorder:  # (a relabelled handle decodes its stored lists)
                    assert np.array_equal(g.decode(0, n), oe), mask
                dist = g.sssp(int(srcs[0]))
                assert np.array_equal(dist.view(np.uint32), dref.view(np.uint32)), mask
        g.free()


def test_random_graphs_many_shapes(efg):
    rng = np.random.default_rng(21)
    for t in range(25):
        n = int(rng.integers(1, 5000))
        m = int(rng.integers(0, 20 * n))
        src = rng.integers(0, n, m).astype(np.uint32)
        dst = rng.integers(0, n, m).astype(np.uint32)
        k = int(rng.choice([0, 4, 8, 100, 512]))
        g, ov, oe = _check_decode(efg, n, src, dst, k)
        _check_bfs(g, ov, oe, rng.integers(0, n, 3))
        g.free()


def test_parents_valid(efg):
    n, src, dst = synth.rmat(14, 16, seed=1)
    g = efg.Graph.build(n, src, dst)
    ov, oe = oracle.csr_build(n, src, dst)
    for s in (0, 77):
        d, par, st = g.bfs(s, parent=True, stats=True)
        ref = oracle.bfs(ov, oe, s)
        assert np.array_equal(d, ref)
        reached = d >= 0
        assert par[s] == s
        assert np.all(par[~reached] == 0xFFFFFFFF)
        for v in np.flatnonzero(reached):
            if v == s:
                continue
            p = int(par[v])
            assert d[p] == d[v] - 1
            assert v in oe[ov[p]:ov[p + 1]]
        assert st["vertices_reached"] == reached.sum()
        assert st["edges_traversed"] == int(np.diff(ov)[reached].sum())
    g.free()


def test_stats_levels(efg):
    n, src, dst = synth.rmat(13, 16, seed=2)
    g = efg.Graph.build(n, src, dst)
    ov, oe = oracle.csr_build(n, src, dst)
    d, _, st = g.bfs(0, stats=True)
    ref = oracle.bfs(ov, oe, 0)
    assert st["levels"] == ref.max() + 1
    for L in range(st["levels"]):
        lvl = ref == L
        assert st["level_frontier"][L] == lvl.sum()
        assert st["level_edges"][L] == np.diff(ov)[lvl].sum()
    g.free()


@pytest.mark.slow
def test_c2_rmat24_full_size(efg):
    # BASELINE.json configs[1] at full size, bench launch configuration
    # (degree relabelling + prefix/list skip, as bench.py times it; then the
    # input order and the full decode)
    n, src, dst = synth.config_edges(2)
    ov, oe = oracle.csr_build(n, src, dst)
    deg = np.diff(ov)
    srcs = synth.sources(n, 2, seed=1002, nonisolated_mask=deg > 0)
    refs = {int(s): oracle.bfs(ov, oe, int(s)) for s in np.concatenate([[0], srcs])}
    g = efg.Graph.build(n, src, dst, flags=efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE)
    for s, ref in refs.items():
        assert np.array_equal(g.bfs(s), ref)
    g.set_prefix_skip(False)
    assert np.array_equal(g.bfs(int(srcs[0])), refs[int(srcs[0])])
    g.free()
    g = efg.Graph.build(n, src, dst)
    del src, dst
    for s, ref in refs.items():
        assert np.array_equal(g.bfs(s), ref)
    # decode of sampled vertex ranges (hubs and tail)
    for a, b in [(0, 64), (n // 2, n // 2 + 4096), (n - 5000, n)]:
        assert np.array_equal(g.decode(a, b), oe[ov[a]:ov[b]])
    g.free()


def test_graph_and_host_level_loops_agree(efg):
    n, src, dst = synth.rmat(13, 16, seed=7)
    g = efg.Graph.build(n, src, dst)
    ov, oe = oracle.csr_build(n, src, dst)
    for s in (0, 3, 4000):
        ref = oracle.bfs(ov, oe, s)
        g.set_level_loop(False)
        d1, _, st1 = g.bfs(s, stats=True)
        g.set_level_loop(True)
        d2, _, st2 = g.bfs(s, stats=True)
        assert np.array_equal(d1, ref) and np.array_equal(d2, ref)
        assert st1["levels"] == st2["levels"] == ref.max() + 1
        assert np.array_equal(st1["level_edges"], st2["level_edges"])
        assert st1["edges_traversed"] == st2["edges_traversed"]
        assert st1["vertices_reached"] == (ref >= 0).sum()
    g.free()


def test_long_path_many_levels(efg):
    # more levels than the per-level statistics buffer (graph-mode device loop)
    n = 6000
    src = np.arange(n - 1, dtype=np.uint32)
    g = efg.Graph.build(n, src, src + 1)
    d, _, st = g.bfs(0, stats=True, level_cap=16)
    assert np.array_equal(d, np.arange(n))
    assert st["levels"] == n and st["vertices_reached"] == n
    g.free()


@pytest.mark.parametrize("plen", [1, 2, 13, 14, 15, 16, 125, 126, 127, 128, 300])
def test_host_depth_transfer_levels_boundary(efg, plen):
    """Host depth arrays cross PCIe as 4 bits per vertex while the BFS has
    fewer than 15 levels, as 1 byte while every depth fits [-1, 126], else as
    int32: paths around both boundaries, plus unreached vertices (-1)."""
    n = 5000
    src = np.arange(plen - 1, dtype=np.uint32)
    g = efg.Graph.build(n, src, src + 1)
    d, _, st = g.bfs(0, stats=True)
    ref = np.full(n, -1, np.int32)
    ref[:plen] = np.arange(plen)
    assert np.array_equal(d, ref)
    assert st["d2h_bytes"] == ((n + 7) // 8 * 4 if plen < 15 else n if plen < 127 else 4 * n)
    g.free()


def test_reorder_degree_bfs_in_input_ids(efg):
    n, src, dst = synth.rmat(14, 16, seed=11)
    g = efg.Graph.build(n, src, dst, flags=efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE)
    ov, oe = oracle.csr_build(n, src, dst)
    # decode describes the relabelled graph
    p = g.perm()
    new_of_old = np.empty(n, np.uint32)
    new_of_old[p] = np.arange(n, dtype=np.uint32)
    rv, re_ = oracle.csr_build(n, new_of_old[src], new_of_old[dst])
    assert np.array_equal(g.decode(0, n), re_)
    # traversal inputs and outputs are in input ids
    _check_bfs(g, ov, oe, [0, 1, 5, n - 1, 4321])
    for s in (0, 99):
        d, par, _ = g.bfs(s, parent=True, stats=True)
        assert np.array_equal(d, oracle.bfs(ov, oe, s))
        assert par[s] == s
        for v in np.flatnonzero(d > 0)[:2000]:
            pv = int(par[v])
            assert d[pv] == d[v] - 1 and v in oe[ov[pv]:ov[pv + 1]]
    g.free()


def test_hot_snapshot_boundary(efg):
    # graph larger than the shared-memory hot range (32,768 ids): probes on both sides
    n, src, dst = synth.rmat(20, 8, seed=12)
    for flags in (efg.EFG_DEFAULT_FLAGS, efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE):
        g = efg.Graph.build(n, src, dst, flags=flags)
        ov, oe = oracle.csr_build(n, src, dst)
        _check_bfs(g, ov, oe, [0, 32767, 32768, 917504, n - 1])
        g.free()


@pytest.mark.parametrize("world", [1, 2, 3, 4])
def test_partitioned_bfs_simulated_ranks(efg, world):
    """the 1-D partitioned kernels (row-range handles, pack /
    OR-reduce / unpack, owned-row frontiers) with the transport emulated in
    one process; every rank's depth must equal the oracle's."""
    import torch
    from paper_conf_ipps_gerak23_b200.dist import simulated_partitioned_bfs
    n, src, dst = synth.rmat(14, 16, seed=13)
    ov, oe = oracle.csr_build(n, src, dst)
    for flags in (efg.EFG_DEFAULT_FLAGS, efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE):
        whole = efg.Graph.build(n, src, dst, flags=flags, device=-1)
        vlist, _, offsets, _ = whole.export()
        bounds = efg.partition(vlist, offsets, world)
        whole.free()
        graphs = [efg.Graph.build(n, src, dst, flags=flags,
                                  rows=(int(bounds[r]), int(bounds[r + 1]))) for r in range(world)]
        for s in (0, 3, 9999):
            depths = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(world)]
            simulated_partitioned_bfs(graphs, s, depths, bounds,
                                      lambda k: torch.zeros(k, dtype=torch.int32, device="cuda"))
            torch.cuda.synchronize()
            ref = oracle.bfs(ov, oe, s)
            for d in depths:
                assert np.array_equal(d.cpu().numpy(), ref)
        for g in graphs:
            g.free()


@pytest.mark.parametrize("world", [1, 2, 3, 4])
def test_partitioned_bfs_peer_exchange_simulated_ranks(efg, world):
    """SURVEY §8(e) over peer memory (efg_peer_* / efg_xchg_peer): the owner
    OR-reduce + broadcast and the cross-rank barriers run in the library's
    kernels; here the ranks share one device (regions mapped by address, one
    non-blocking stream per rank).  Every rank's depth must equal the oracle's,
    over several BFS on the same mapping (barrier epochs keep counting)."""
    import torch
    from paper_conf_ipps_gerak23_b200.dist import simulated_peer_setup, simulated_partitioned_bfs_peer
    n, src, dst = synth.rmat(14, 16, seed=13)
    ov, oe = oracle.csr_build(n, src, dst)
    for flags in (efg.EFG_DEFAULT_FLAGS, efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE):
        whole = efg.Graph.build(n, src, dst, flags=flags, device=-1)
        vlist, _, offsets, _ = whole.export()
        bounds = efg.partition(vlist, offsets, world)
        whole.free()
        streams = [torch.cuda.Stream() for _ in range(world)]
        graphs = [efg.Graph.build(n, src, dst, flags=flags, stream=streams[r].cuda_stream,
                                  rows=(int(bounds[r]), int(bounds[r + 1]))) for r in range(world)]
        simulated_peer_setup(graphs, bounds)
        sparse = dense = 0
        for s in (0, 3, 9999, n - 1):
            depths = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(world)]
            torch.cuda.synchronize()
            counts = simulated_partitioned_bfs_peer(graphs, s, depths)
            torch.cuda.synchronize()
            ref = oracle.bfs(ov, oe, s)
            for d in depths:
                assert np.array_equal(d.cpu().numpy(), ref)
            sts = [g.bfs_end() for g in graphs]
            assert len({st["xchg_sparse_levels"] for st in sts}) == 1  # one decision on every rank
            sparse += sts[0]["xchg_sparse_levels"]
            dense += len(counts) - sts[0]["xchg_sparse_levels"]
        if world > 1:  # both exchange paths ran (small levels sparse, the heavy ones dense)
            assert sparse > 0 and dense > 0, (sparse, dense)
        for g in graphs:
            g.free()


def test_peer_exchange_errors(efg):
    n, src, dst = synth.rmat(10, 8, seed=3)
    g = efg.Graph.build(n, src, dst)
    bounds = np.array([0, n], np.uint64)
    with pytest.raises(efg.EFGError):
        g.xchg_peer()                       # before efg_peer_open
    with pytest.raises(efg.EFGError):
        g.peer_open(0, bounds, regions=[0])  # before efg_peer_alloc
    reg, h = g.peer_alloc(1)
    assert reg != 0 and len(h) == 64
    with pytest.raises(efg.EFGError):
        g.peer_open(0, np.array([0, n - 1], np.uint64), regions=[reg])  # bounds do not span [0, n)
    g.peer_open(0, bounds, regions=[reg])
    g.free()


@pytest.mark.parametrize("reorder", [False, True])
def test_sssp_bit_exact_vs_dijkstra(efg, reorder):
    """NEXT-1: fp32 frontier Bellman-Ford == fp32 Dijkstra bit for bit (C20)."""
    n, src, dst = synth.rmat(13, 16, seed=21)
    w_in = synth.weights(src, dst, seed=2000 + 1)
    flags = efg.EFG_DEFAULT_FLAGS | (efg.EFG_REORDER_DEGREE if reorder else 0)
    g = efg.Graph.build(n, src, dst, weights=w_in, flags=flags)
    ov, oe = oracle.csr_build(n, src, dst)
    u = np.repeat(np.arange(n, dtype=np.uint32), np.diff(ov).astype(np.int64))
    w_csr = synth.weights(u, oe, seed=2000 + 1)  # symmetric pair function -> CSR-order weights
    for s in (0, 17, 4000):
        got = g.sssp(s)
        ref = oracle.sssp(ov, oe, w_csr, s)
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32)), s
    g.free()


def test_sssp_requires_weights(efg):
    n, src, dst = synth.rmat(10, 8, seed=1)
    g = efg.Graph.build(n, src, dst)
    with pytest.raises(efg.EFGError):
        g.sssp(0)
    g.free()


@pytest.mark.parametrize("reorder", [False, True])
def test_pagerank_vs_fp64_oracle(efg, reorder):
    """NEXT-2 (P:185, 50 iterations P:201): within 1e-6 relative L1 of the fp64 oracle."""
    n, src, dst = synth.rmat(14, 16, seed=22)
    flags = efg.EFG_DEFAULT_FLAGS | (efg.EFG_REORDER_DEGREE if reorder else 0)
    g = efg.Graph.build(n, src, dst, flags=flags)
    ov, oe = oracle.csr_build(n, src, dst)
    ref = oracle.pagerank(ov, oe, 0.85, 50)
    for pull in (True, False):  # gather over own lists / push along every edge
        g.set_pagerank_pull(pull)
        got = g.pagerank(0.85, 50)
        rel = np.abs(got - ref).sum() / np.abs(ref).sum()
        assert rel < 1e-6, (pull, rel)
        assert abs(got.sum() - 1.0) < 1e-9
    g.free()


def test_pagerank_directed_uses_push(efg):
    """A directed handle's lists are out-lists only: PageRank pushes (pull option ignored)."""
    n, src, dst = synth.rmat(12, 8, seed=23)
    g = efg.Graph.build(n, src, dst, flags=efg.EFG_DEDUP | efg.EFG_DROP_SELF_LOOPS)
    ov, oe = oracle.csr_build(n, src, dst, symmetrize=False)
    got = g.pagerank(0.85, 50)
    ref = oracle.pagerank(ov, oe, 0.85, 50)
    assert np.abs(got - ref).sum() / np.abs(ref).sum() < 1e-6
    g.free()


@pytest.mark.slow
def test_pagerank_c2_full_size(efg):
    """NEXT-2 at its BASELINE config (configs[1]: RMAT-24/ef16, BFS and PageRank):
    50 iterations within 1e-6 relative L1 of the fp64 oracle, pull (gather) and
    push both, on the bench's degree-relabelled build."""
    n, src, dst = synth.config_edges(2)
    ov, oe = oracle.csr_build(n, src, dst)
    ref = oracle.pagerank(ov, oe, 0.85, 50)
    g = efg.Graph.build(n, src, dst, flags=efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE)
    del src, dst
    for pull in (True, False):
        g.set_pagerank_pull(pull)
        got = g.pagerank(0.85, 50)
        rel = np.abs(got - ref).sum() / np.abs(ref).sum()
        assert rel < 1e-6, (pull, rel)
    g.free()
