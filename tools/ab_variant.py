"""Same-graph A/B of expand-kernel variants (EFG_OPT_EXPAND_VARIANT masks) and
of the prefix skip, on one BASELINE config: build once, then alternate the
variants over the same sources (graph-mode BFS, CUDA events), and check that
every variant's depths equal the first variant's.  Per-level expand times come
from a host-loop pass per variant.

  python tools/ab_variant.py --config 3 --masks 0,3,1,2 --sources 8 --rounds 2
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_ipps_gerak23_b200 as efg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=3)
ap.add_argument("--scale", type=int, default=None)
ap.add_argument("--masks", default="0,3")
ap.add_argument("--sources", type=int, default=8)
ap.add_argument("--rounds", type=int, default=2)
ap.add_argument("--reorder", default="degree")
ap.add_argument("--levels", action="store_true")
a = ap.parse_args()
masks = [int(x) for x in a.masks.split(",")]

sg = synth.config_stream(a.config, scale_override=a.scale)
n = sg.n
flags = efg.EFG_DEFAULT_FLAGS | (efg.EFG_REORDER_DEGREE if a.reorder == "degree" else 0)
stream = torch.cuda.Stream()
g = efg.Graph.build_stream(n, sg.m, sg.fn, sg.user, stream=stream.cuda_stream, flags=flags,
                           n_threads=os.cpu_count() or 1)
vl = g.export()[0]
perm = g.perm()
deg = np.empty(n, np.int64)
deg[perm] = np.diff(vl).astype(np.int64)
srcs = synth.sources(n, a.sources + 2, seed=1000 + a.config, nonisolated_mask=deg > 0)
depth = torch.empty(n, dtype=torch.int32, device="cuda")
edges = 0
for s in srcs[2:]:
    _, _, st = g.bfs(int(s), depth=depth, stats=True)
    edges += st["edges_traversed"]
ref = {}
res = {m: [] for m in masks}
lv = {}
for r in range(a.rounds):
    for m in masks:
        g.set_expand_variant(m)
        with torch.cuda.stream(stream):
            for s in srcs[:2]:
                g.bfs(int(s), depth=depth)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        with torch.cuda.stream(stream):
            for s in srcs[2:]:
                g.bfs(int(s), depth=depth)
        e1.record(stream)
        torch.cuda.synchronize()
        res[m].append(edges / (e0.elapsed_time(e1) * 1e-3) / 1e9)
        if r == 0:
            for s in srcs[2:4]:
                d = g.bfs(int(s))
                key = int(s)
                if key not in ref:
                    ref[key] = d
                elif not np.array_equal(ref[key], d):
                    print(json.dumps({"mask": m, "source": key, "MISMATCH": int((ref[key] != d).sum())}))
                    sys.exit(1)
            if a.levels:
                g.set_level_loop(True)
                _, _, st = g.bfs(int(srcs[2]), depth=depth, stats=True)
                g.set_level_loop(False)
                lv[m] = [round(float(x), 3) for x in st["level_expand_ms"]]
print(json.dumps({"config": a.config, "edges_per_run": edges,
                  "gteps": {m: [round(x, 1) for x in v] for m, v in res.items()},
                  "level_expand_ms": lv, "depth_agree": True}))
