"""Full-size parity of a BASELINE.json config (C3 / C4: too large for the
default GPU test run): the CUDA path (bench.py's build — streamed from the
generator, degree relabelling or another id order, prefix/list skip) against
the oracle on the same seeded graph.

  python tests/verify_full.py --config 3 --sources 3 > profiles/r02_verify_c3.json
  python tests/verify_full.py --config 4 --sources 2 --order random
  python tests/verify_full.py --config 4 --sources 1 --sssp

Phase 1 runs the GPU path and keeps only its outputs; phase 2 builds the
oracle's own CSR from the generator's edge list (oracle.csr_build, no product
code) and compares: BFS depth bit-exact vs the oracle's FIFO BFS; with --sssp,
fp32 distances bit-exact vs the oracle's fp32 Dijkstra (reading C20) from the
same sources.  The phases never hold both graphs, so C4 (~7 B directed edges)
fits a 196 GB host.  Prints one JSON line.
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
ap.add_argument("--order", default="degree", choices=["degree", "locality", "random"],
                help="degree relabelling, the generator's order, or a random permutation (P:248-258)")
ap.add_argument("--sssp", action="store_true", help="also SSSP (weighted build in the generator's order)")
a = ap.parse_args()
permute = True if a.order == "random" else None
flags = efg.EFG_DEFAULT_FLAGS | (efg.EFG_REORDER_DEGREE if a.order == "degree" else 0)
nthr = os.cpu_count() or 1

# ---- phase 1: the CUDA path ----
sg = synth.config_stream(a.config, permute=permute)
n = sg.n
t0 = time.time()
g = efg.Graph.build_stream(n, sg.m, sg.fn, sg.user, flags=flags, n_threads=nthr)
t_build = time.time() - t0
vl = g.export()[0]
perm = g.perm()
deg = np.empty(n, np.int64)
deg[perm] = np.diff(vl).astype(np.int64)
m_dir = int(vl[-1])
del vl, perm
srcs = synth.sources(n, a.sources, seed=1000 + a.config, nonisolated_mask=deg > 0)
got = {int(s): g.bfs(int(s)) for s in srcs}
g.free()
got_sssp = {}
if a.sssp:
    gw = efg.Graph.build_stream(n, sg.m, sg.fn, sg.user, weighted=True, n_threads=nthr)
    for s in srcs:
        got_sssp[int(s)] = gw.sssp(int(s))
    gw.free()

# ---- phase 2: the oracle ----
t0 = time.time()
_, src, dst = synth.config_edges(a.config, permute=permute)
t_gen = time.time() - t0
t0 = time.time()
ov, oe = oracle.csr_build(n, src, dst)
t_csr = time.time() - t0
del src, dst
odeg = np.diff(ov)
res = []
for s in srcs:
    t0 = time.time()
    ref = oracle.bfs(ov, oe, int(s))
    t_or = time.time() - t0
    d = got[int(s)]
    ok = bool(np.array_equal(d, ref))
    r = {"source": int(s), "bit_exact": ok, "reached": int((ref >= 0).sum()),
         "levels": int(ref.max()) + 1, "edges": int(odeg[ref >= 0].sum()),
         "oracle_bfs_s": round(t_or, 2), "mismatches": 0 if ok else int((d != ref).sum())}
    res.append(r)
sres = []
if a.sssp:
    u = np.repeat(np.arange(n, dtype=np.uint32), odeg.astype(np.int64))
    w_csr = synth.weights(u, oe, seed=2000 + a.config)  # symmetric pair weights in CSR order (C20)
    del u
    for s in srcs:
        t0 = time.time()
        ref = oracle.sssp(ov, oe, w_csr, int(s))
        t_or = time.time() - t0
        d = got_sssp[int(s)]
        ok = bool(np.array_equal(d.view(np.uint32), ref.view(np.uint32)))
        sres.append({"source": int(s), "bit_exact": ok, "reached": int(np.isfinite(ref).sum()),
                     "oracle_dijkstra_s": round(t_or, 1),
                     "mismatches": 0 if ok else int((d.view(np.uint32) != ref.view(np.uint32)).sum())})
line = {"config": synth.CONFIGS[a.config]["name"], "order": a.order, "n": int(n), "samples": int(sg.m),
        "m_directed": int(ov[-1]), "m_directed_efg": m_dir,
        "check": "BFS depth bit-exact vs oracle FIFO BFS over the oracle CSR"
                 + ("; SSSP fp32 distances bit-exact vs oracle fp32 Dijkstra" if a.sssp else ""),
        "efg_build_s": round(t_build, 1), "gen_s": round(t_gen, 1), "oracle_csr_s": round(t_csr, 1),
        "sources": res, "sssp": sres or None,
        "host_peak_rss_gb": round(__import__("resource").getrusage(__import__("resource").RUSAGE_SELF).ru_maxrss
                                  * 1024 / 1e9, 1),
        "all_exact": all(r["bit_exact"] for r in res + sres) and m_dir == int(ov[-1])}
print(json.dumps(line))
