"""GPU tests of the C-ABI boundary's edge cases (include/efg.h):

  * any forward-pointer quantum k (§VI-C) gives the oracle's lists and
    depths: k = 0 (no pointers) and k > 512 have chunks whose lower fields do
    not fit the expand kernel's staging buffer, and a small k with a large hub
    overflows the descriptor's chunk-index field — the device copy re-samples
    its pointers every 512 elements (efg_info_t.device_quantum, reading R3);
  * a hub list whose last k-chunks are so sparse that four of them span more
    than 2^16 upper-bit words (the expand producer must not pack the batch's
    word offsets into 16 bits);
  * row-range (partitioned) handles: efg_bfs is collective over the peer
    exchange and refuses to run without it; SSSP / PageRank are not offered.
Every traversal result is compared bit-exactly with the CPU oracle.
"""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def efg(cuda_ok):
    import paper_conf_ipps_gerak23_b200 as m
    return m


def _decode_bfs_exact(g, n, ov, oe, sources):
    got = g.decode(0, n)
    assert got.size == oe.size and np.array_equal(got, oe)
    for s in sources:
        assert np.array_equal(g.bfs(int(s)), oracle.bfs(ov, oe, int(s))), s


@pytest.mark.parametrize("k", [0, 4096, 1000])
def test_quantum_outside_device_range_rmat18(efg, k):
    """RMAT-18 (hubs of several thousand neighbours): with k = 0 or k > 512 a
    single chunk's lower fields exceed a staging buffer; the device copy uses
    512-element chunks and the results stay exact."""
    n, src, dst = synth.rmat(18, 16, seed=5)
    ov, oe = oracle.csr_build(n, src, dst)
    g = efg.Graph.build(n, src, dst, k=k)
    assert g.info["fwd_quantum"] == k
    assert g.info["device_quantum"] == 512
    # the host arrays keep the caller's k: forward-pointer bytes = 4 floor(deg/k)
    deg = np.diff(ov)
    assert g.info["fwd_bytes"] == (0 if k == 0 else int((4 * (deg // k)).sum()))
    deg_src = synth.sources(n, 4, 1005, deg > 0)
    _decode_bfs_exact(g, n, ov, oe, np.concatenate([[0], deg_src]))
    g.set_level_loop(True)
    assert np.array_equal(g.bfs(0), oracle.bfs(ov, oe, 0))
    g.free()


def test_small_quantum_huge_hub_chunk_index(efg):
    """k = 8 and a star of 2^21 + 5 leaves: ceil(deg/k) >= 2^18 chunks would
    not fit the descriptor's chunk-index field -> device quantum 512."""
    leaves = (1 << 21) + 5
    n = leaves + 1
    src = np.zeros(leaves, np.uint32)
    dst = np.arange(1, n, dtype=np.uint32)
    ov, oe = oracle.csr_build(n, src, dst)
    g = efg.Graph.build(n, src, dst, k=8)
    assert g.info["device_quantum"] == 512
    _decode_bfs_exact(g, n, ov, oe, [0, 1, n - 1])
    g.free()
    # a small k where every list fits keeps the format's quantum on the device
    g = efg.Graph.build(n, src[:1000], dst[:1000], k=8)
    assert g.info["device_quantum"] == 8
    g.free()


def test_sparse_hub_tail_batch_over_2e16_words(efg):
    """Hub of 2^21 neighbours on n = 2^22: l = 0 (u < 2 deg), a dense head and a
    tail of 1536 ids spaced 1367 apart, so the last three 512-element chunks
    span > 2^16 upper-bit words.  From the hub as source (work position 0,
    544 work units per chunk, 2048 per tile) those three chunks form one tile,
    hence one producer batch, whose word offsets overflow 16 bits."""
    n = 1 << 22
    hub = n - 1
    u = n - 2
    tail = (u - 1367 * np.arange(1535, -1, -1)).astype(np.uint32)
    head = np.arange(0, (1 << 21) - 1536, dtype=np.uint32)
    assert head[-1] < tail[0]
    nb = np.concatenate([head, tail])
    rng = np.random.default_rng(3)
    extra_s = rng.integers(0, n, 200_000).astype(np.uint32)
    extra_d = rng.integers(0, n, 200_000).astype(np.uint32)
    keep = (extra_s != hub) & (extra_d != hub)  # the hub's list is exactly nb
    extra_s, extra_d = extra_s[keep], extra_d[keep]
    src = np.concatenate([np.full(nb.size, hub, np.uint32), extra_s])
    dst = np.concatenate([nb, extra_d])
    ov, oe = oracle.csr_build(n, src, dst)
    lst = oe[ov[hub]:ov[hub + 1]]
    u, d = int(lst[-1]), lst.size
    assert u < 2 * d  # l = 0
    # upper bits of the last three chunks: span of their high parts + elements
    span_words = (int(lst[-1]) - int(lst[d - 1536]) + 1536) // 32
    assert span_words > (1 << 16)
    g = efg.Graph.build(n, src, dst)
    _decode_bfs_exact(g, n, ov, oe, [hub, 0, int(tail[-1])])
    g.free()


def _partition(efg, n, src, dst, world, flags):
    whole = efg.Graph.build(n, src, dst, flags=flags, device=-1)
    vlist, _, offsets, _ = whole.export()
    bounds = efg.partition(vlist, offsets, world)
    whole.free()
    return bounds


def test_partitioned_handle_errors(efg):
    n, src, dst = synth.rmat(12, 8, seed=3)
    bounds = _partition(efg, n, src, dst, 2, efg.EFG_DEFAULT_FLAGS)
    g = efg.Graph.build(n, src, dst, rows=(int(bounds[0]), int(bounds[1])),
                        weights=synth.weights(src, dst, 7))
    with pytest.raises(efg.EFGError) as e:
        g.bfs(0)                       # collective BFS needs the peer exchange
    assert e.value.status == 7         # EFG_ESTATE
    with pytest.raises(efg.EFGError) as e:
        g.sssp(0)
    assert e.value.status == 6         # EFG_ENOTSUP
    with pytest.raises(efg.EFGError) as e:
        g.pagerank()
    assert e.value.status == 6
    g.free()


@pytest.mark.parametrize("world", [2, 3])
def test_collective_bfs_on_partitioned_handles(efg, world):
    """efg_bfs on row-range handles after efg_peer_open: one collective call per
    rank (enqueue-only form: device depth, no stats), the level loop a CUDA
    graph per rank that stops on the device when the global new count is 0.
    Ranks share one device here (regions by address, one non-blocking stream
    each).  Every rank's depth equals the oracle's."""
    import torch
    from paper_conf_ipps_gerak23_b200.dist import simulated_peer_setup
    n, src, dst = synth.rmat(14, 16, seed=13)
    ov, oe = oracle.csr_build(n, src, dst)
    for flags in (efg.EFG_DEFAULT_FLAGS, efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE):
        bounds = _partition(efg, n, src, dst, world, flags)
        streams = [torch.cuda.Stream() for _ in range(world)]
        graphs = [efg.Graph.build(n, src, dst, flags=flags, stream=streams[r].cuda_stream,
                                  rows=(int(bounds[r]), int(bounds[r + 1]))) for r in range(world)]
        simulated_peer_setup(graphs, bounds)
        for s in (0, 3, 9999, n - 1):
            depths = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(world)]
            torch.cuda.synchronize()
            for g, d in zip(graphs, depths):
                g.bfs(s, depth=d)
            torch.cuda.synchronize()
            ref = oracle.bfs(ov, oe, s)
            for d in depths:
                assert np.array_equal(d.cpu().numpy(), ref), s
        # the stepwise calls still work on the same mapping (shared epoch counter)
        from paper_conf_ipps_gerak23_b200.dist import simulated_partitioned_bfs_peer
        depths = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(world)]
        simulated_partitioned_bfs_peer(graphs, 5, depths)
        torch.cuda.synchronize()
        for d in depths:
            assert np.array_equal(d.cpu().numpy(), oracle.bfs(ov, oe, 5))
        for g in graphs:
            g.free()


@pytest.mark.parametrize("reorder", [False, True])
def test_host_resident_out_of_core(efg, reorder):
    """EFG_HOST_RESIDENT (out-of-core, P:34 / P:222): the EF data stays in
    pinned host memory mapped into the device; every traversal reads it over
    the host link and gives the oracle's results."""
    n, src, dst = synth.rmat(15, 16, seed=31)
    w = synth.weights(src, dst, 2031)
    flags = efg.EFG_DEFAULT_FLAGS | efg.EFG_HOST_RESIDENT | (efg.EFG_REORDER_DEGREE if reorder else 0)
    g = efg.Graph.build(n, src, dst, flags=flags, weights=w)
    assert g.info["data_location"] == 1
    ov, oe = oracle.csr_build(n, src, dst)
    if not reorder:
        assert np.array_equal(g.decode(0, n), oe)
    deg = np.diff(ov)
    for s in np.concatenate([[0], synth.sources(n, 3, 1031, deg > 0)]):
        assert np.array_equal(g.bfs(int(s)), oracle.bfs(ov, oe, int(s)))
    u = np.repeat(np.arange(n, dtype=np.uint32), deg.astype(np.int64))
    w_csr = synth.weights(u, oe, seed=2031)
    got = g.sssp(3)
    assert np.array_equal(got.view(np.uint32), oracle.sssp(ov, oe, w_csr, 3).view(np.uint32))
    pr = g.pagerank(0.85, 50)
    ref = oracle.pagerank(ov, oe, 0.85, 50)
    assert np.abs(pr - ref).sum() / np.abs(ref).sum() < 1e-6
    g.free()
    g = efg.Graph.build(n, src, dst)
    assert g.info["data_location"] == 0
    g.free()
