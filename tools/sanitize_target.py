"""Workload for tools/gpu_sanitize.sh (compute-sanitizer): every traversal mode
on small graphs, each result checked against the oracle so a run that the
sanitizer slows down still proves the same answers."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import oracle  # noqa: E402
import synth  # noqa: E402
import paper_conf_ipps_gerak23_b200 as efg  # noqa: E402

n, src, dst = synth.rmat(12, 16, seed=1)
ov, oe = oracle.csr_build(n, src, dst)
w = synth.weights(src, dst, 2001)
u = np.repeat(np.arange(n, dtype=np.uint32), np.diff(ov).astype(np.int64))
w_csr = synth.weights(u, oe, seed=2001)
for flags in (efg.EFG_DEFAULT_FLAGS, efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE,
              efg.EFG_DEFAULT_FLAGS | efg.EFG_HOST_RESIDENT):
    g = efg.Graph.build(n, src, dst, flags=flags, weights=w)
    if not flags & efg.EFG_REORDER_DEGREE:
        assert np.array_equal(g.decode(0, n), oe)
    # host-driven level loop only: under the sanitizer, launches of the graph
    # with the device-side WHILE loop fail on their first kernel node (the
    # graph loop is covered by every GPU test without the sanitizer)
    g.set_level_loop(True)
    for s in (0, 5):
        assert np.array_equal(g.bfs(s), oracle.bfs(ov, oe, s))
    d, par, _ = g.bfs(7, parent=True, stats=True)
    assert np.array_equal(d, oracle.bfs(ov, oe, 7))
    assert np.array_equal(g.sssp(3).view(np.uint32), oracle.sssp(ov, oe, w_csr, 3).view(np.uint32))
    pr = g.pagerank(0.85, 20)
    ref = oracle.pagerank(ov, oe, 0.85, 20)
    assert np.abs(pr - ref).sum() / np.abs(ref).sum() < 1e-6
    g.free()
# The peer exchange with device barriers is left out (the sanitizer
# serialises kernel launches, so one rank's barrier kernel would wait for a
# rank that cannot start); the host-sequenced form has no such wait: two
# simulated ranks in this process, the phases issued rank by rank (dense and
# sparse levels both occur on this graph).
import torch  # noqa: E402
from paper_conf_ipps_gerak23_b200.dist import simulated_peer_setup  # noqa: E402

world = 2
whole = efg.Graph.build(n, src, dst, device=-1)
vl, _, of, _ = whole.export()
bounds = efg.partition(vl, of, world)
whole.free()
streams = [torch.cuda.Stream() for _ in range(world)]
gs = [efg.Graph.build(n, src, dst, stream=streams[r].cuda_stream, rows=(int(bounds[r]), int(bounds[r + 1])))
      for r in range(world)]
simulated_peer_setup(gs, bounds)
for s in (0, 5):
    depths = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(world)]
    for g, d in zip(gs, depths):
        g.bfs_begin(s, d)
    while True:
        for g in gs:
            g.bfs_expand()
        for phase in (0, 1, 2):
            for g in gs:
                g.xchg_peer_phase(phase)  # synchronises its stream
        news = [g.bfs_finish_level() for g in gs]
        assert len(set(news)) == 1
        if news[0] == 0:
            break
    torch.cuda.synchronize()
    for d in depths:
        assert np.array_equal(d.cpu().numpy(), oracle.bfs(ov, oe, s))
    assert len({g.bfs_end()["xchg_sparse_levels"] for g in gs}) == 1
for g in gs:
    g.free()
print("sanitize_target: all traversals match the oracle")
