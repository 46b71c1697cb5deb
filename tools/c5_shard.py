"""BASELINE configs[4] (C5: RMAT scale 29, edgefactor 32, permuted ids, 8 GPUs,
1-D partition): build ONE rank's shard with efg_build_stream — the edges come
from the counter-based generator in two chunked passes, the builder keeps only
the owned rows' adjacency — and report its size, build time and
the peak resident memory of the process.

  python tools/c5_shard.py --rank 0 --world 8 [--device 0] > profiles/r02_c5_shard0.json
"""
import argparse
import json
import os
import resource
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
import paper_conf_ipps_gerak23_b200 as efg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--rank", type=int, default=0)
ap.add_argument("--world", type=int, default=8)
ap.add_argument("--scale", type=int, default=None)
ap.add_argument("--device", type=int, default=-1, help="-1: host-only handle")
a = ap.parse_args()
sg = synth.config_stream(5, scale_override=a.scale)
n = sg.n
# equal 64-aligned vertex ranges: ids are permuted (C5), so degrees are spread evenly
bounds = [min(n, (n * r // a.world + 63) // 64 * 64) for r in range(a.world)] + [n]
lo, hi = bounds[a.rank], bounds[a.rank + 1]
t0 = time.time()
g = efg.Graph.build_stream(n, sg.m, sg.fn, sg.user, device=a.device, rows=(lo, hi),
                           n_threads=os.cpu_count() or 1)
t = time.time() - t0
i = g.info
rss = resource.getrusage(resource.RUSAGE_SELF).ru_maxrss * 1024 / 1e9
print(json.dumps({"config": "rmat29_ef32" if a.scale is None else f"rmat{a.scale}_ef32", "n": n, "samples": sg.m,
                  "world": a.world, "rank": a.rank, "rows": [lo, hi],
                  "shard_directed_edges": i["m"], "shard_ef_data_bytes": i["data_bytes"],
                  "shard_ef_bytes_per_edge": i["data_bytes"] / max(i["m"], 1),
                  "device_bytes": i["device_bytes"], "data_location": i["data_location"],
                  "build_s": round(t, 1), "host_peak_rss_gb": round(rss, 1), "host_cores": os.cpu_count(),
                  "note": "two generator passes over all samples; only rows [lo, hi) materialised"}))
g.free()
