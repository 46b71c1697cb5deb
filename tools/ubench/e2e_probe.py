"""Where does the e2e (host depth array) time go on C2?  Per-BFS ms for:
(a) device depth, back-to-back; (b) device depth, synchronise after each;
(c) host pinned depth with statistics; (d) host pinned depth without."""
import sys, time
import numpy as np
import torch
sys.path.insert(0, ".")
import synth
import paper_conf_ipps_gerak23_b200 as efg

n, src, dst = synth.config_edges(2)
g = efg.Graph.build(n, src, dst, flags=efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE, n_threads=16)
deg = np.diff(g.export()[0])[np.argsort(g.perm())] if False else None
srcs = [int(s) for s in synth.sources(n, 8, seed=1002)]
dd = torch.empty(n, dtype=torch.int32, device="cuda")
hd = torch.empty(n, dtype=torch.int32, pin_memory=True)
for s in srcs[:3]:
    g.bfs(s, depth=dd); g.bfs(s, depth=hd)
torch.cuda.synchronize()
def run(label, fn):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    for s in srcs: fn(s)
    torch.cuda.synchronize(); t = (time.perf_counter() - t0) / len(srcs) * 1e3
    print(f"{label}: {t:.3f} ms/BFS", flush=True)
for _ in range(2):
    run("(a) device, back-to-back", lambda s: g.bfs(s, depth=dd))
    run("(b) device, sync each", lambda s: (g.bfs(s, depth=dd), torch.cuda.synchronize()))
    run("(c) host, stats", lambda s: g.bfs(s, depth=hd, stats=True))
    run("(d) host, no stats", lambda s: g.bfs(s, depth=hd))
