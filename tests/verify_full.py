"""Full-size parity of a BASELINE.json config (C3 / C4: too large for the
default GPU test run): the CUDA path (bench.py's build: degree relabelling,
prefix/list skip) against the oracle on the same seeded graph.

  python tests/verify_full.py --config 3 --sources 3 > profiles/r1_verify_c3.json

For every sampled source: depth bit-exact vs the oracle's FIFO BFS over its
own CSR (oracle.csr_build, no product code).  Prints one JSON line.
"""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import synth  # noqa: E402
import paper_conf_ipps_gerak23_b200 as efg  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=3)
ap.add_argument("--sources", type=int, default=3)
a = ap.parse_args()
t0 = time.time()
n, src, dst = synth.config_edges(a.config)
t_gen = time.time() - t0
t0 = time.time()
ov, oe = oracle.csr_build(n, src, dst)
t_csr = time.time() - t0
deg = np.diff(ov)
srcs = synth.sources(n, a.sources, seed=1000 + a.config, nonisolated_mask=deg > 0)
t0 = time.time()
g = efg.Graph.build(n, src, dst, flags=efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE,
                    n_threads=os.cpu_count() or 1)
t_build = time.time() - t0
del src, dst
res = []
for s in srcs:
    t0 = time.time()
    ref = oracle.bfs(ov, oe, int(s))
    t_or = time.time() - t0
    got = g.bfs(int(s))
    ok = bool(np.array_equal(got, ref))
    res.append({"source": int(s), "bit_exact": ok, "reached": int((ref >= 0).sum()),
                "levels": int(ref.max()) + 1, "edges": int(deg[ref >= 0].sum()),
                "oracle_bfs_s": round(t_or, 2),
                "mismatches": 0 if ok else int((got != ref).sum())})
g.free()
print(json.dumps({"config": synth.CONFIGS[a.config]["name"], "n": int(n), "m_directed": int(ov[-1]),
                  "check": "depth bit-exact vs oracle FIFO BFS over the oracle CSR",
                  "gen_s": round(t_gen, 1), "oracle_csr_s": round(t_csr, 1), "efg_build_s": round(t_build, 1),
                  "sources": res, "all_exact": all(r["bit_exact"] for r in res)}))
