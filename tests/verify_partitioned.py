"""Simulated multi-GPU parity at scale: W ranks of the 1-D row partition
 on ONE GPU, each rank a row-range handle of the C5 recipe at a
smaller scale (RMAT, edgefactor 32, permuted ids), traversed with
  (a) the stepwise calls and a host-emulated all-to-all / all-gather, and
  (b) the collective efg_bfs over the peer-memory exchange (ranks mapped by
      address, one stream each, level loop on the device),
and compared bit-exactly with the oracle's FIFO BFS over its own CSR.

  python tests/verify_partitioned.py --scale 26 --world 8 --sources 2 > profiles/r02_verify_partitioned_rmat26.json
"""
import argparse
import json
import os
import resource
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import synth  # noqa: E402
import paper_conf_ipps_gerak23_b200 as efg  # noqa: E402
from paper_conf_ipps_gerak23_b200.dist import (simulated_partitioned_bfs, simulated_peer_setup)  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--scale", type=int, default=26)
ap.add_argument("--world", type=int, default=8)
ap.add_argument("--sources", type=int, default=2)
ap.add_argument("--no-peer", action="store_true")
a = ap.parse_args()

import torch  # noqa: E402

# W ranks share one GPU: each rank's persistent frontier grid (its blocks wait
# on each other) is sized to 2 blocks per SM instead of the whole GPU, so that
# the other ranks' one-block exchange barriers can never keep it from being
# co-resident (with real multi-GPU every rank owns its device)
os.environ.setdefault("EFG_FRONTIER_BLOCKS", str(2 * torch.cuda.get_device_properties(0).multi_processor_count))
t0 = time.time()
n, src, dst = synth.config_edges(5, scale_override=a.scale)
t_gen = time.time() - t0
W = a.world
bounds = np.array([min(n, (n * r // W + 63) // 64 * 64) for r in range(W)] + [n], np.uint64)
streams = [torch.cuda.Stream() for _ in range(W)]
t0 = time.time()
graphs = [efg.Graph.build(n, src, dst, stream=streams[r].cuda_stream, rows=(int(bounds[r]), int(bounds[r + 1])),
                          n_threads=os.cpu_count() or 1) for r in range(W)]
t_build = time.time() - t0
shard_edges = [g.info["m"] for g in graphs]
t0 = time.time()
ov, oe = oracle.csr_build(n, src, dst)
t_csr = time.time() - t0
del src, dst
deg = np.diff(ov)
srcs = synth.sources(n, a.sources, seed=1005, nonisolated_mask=deg > 0)
mk = lambda k: torch.zeros(k, dtype=torch.int32, device="cuda")  # noqa: E731
res = []
if not a.no_peer:
    simulated_peer_setup(graphs, bounds)
for s in srcs:
    ref = oracle.bfs(ov, oe, int(s))
    r = {"source": int(s), "reached": int((ref >= 0).sum()), "levels": int(ref.max()) + 1,
         "edges": int(deg[ref >= 0].sum())}
    depths = [torch.empty(n, dtype=torch.int32, device="cuda") for _ in range(W)]
    torch.cuda.synchronize()
    t0 = time.time()
    simulated_partitioned_bfs(graphs, int(s), depths, bounds, mk)
    torch.cuda.synchronize()
    r["stepwise_s"] = round(time.time() - t0, 3)
    r["stepwise_bit_exact"] = all(np.array_equal(d.cpu().numpy(), ref) for d in depths)
    if not a.no_peer:
        for d in depths:
            d.fill_(-7)
        torch.cuda.synchronize()
        t0 = time.time()
        for g, d in zip(graphs, depths):
            g.bfs(int(s), depth=d)  # collective: enqueue-only, every rank's loop on the device
        torch.cuda.synchronize()
        r["collective_peer_s"] = round(time.time() - t0, 3)
        r["collective_peer_bit_exact"] = all(np.array_equal(d.cpu().numpy(), ref) for d in depths)
    res.append(r)
for g in graphs:
    g.free()
ok = all(r["stepwise_bit_exact"] and r.get("collective_peer_bit_exact", True) for r in res)
print(json.dumps({"config": f"rmat{a.scale}_ef32 (C5 recipe, permuted)", "n": n, "world": W, "gpus": 1,
                  "bounds": [int(x) for x in bounds], "shard_directed_edges": shard_edges,
                  "m_directed": int(ov[-1]), "sum_shards_equals_m": sum(shard_edges) == int(ov[-1]),
                  "gen_s": round(t_gen, 1), "shard_builds_s": round(t_build, 1), "oracle_csr_s": round(t_csr, 1),
                  "sources": res, "all_exact": ok and sum(shard_edges) == int(ov[-1]),
                  "host_peak_rss_gb": round(resource.getrusage(resource.RUSAGE_SELF).ru_maxrss * 1024 / 1e9, 1),
                  "note": "all ranks time-share one GPU: times are functional, not multi-GPU performance"}))
