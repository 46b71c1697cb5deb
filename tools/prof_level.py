"""Profile target: one BFS on C2 with the host-driven level loop, so that each
expand launch is a separate kernel ncu can pick by index.

usage (on the GPU box):
  ncu --profile-from-start off --kernel-name regex:expand --launch-skip 1 --launch-count 2 \
      --set full --import-source on --clock-control none -o gpurun_out/prof \
      python tools/prof_level.py [source] [reorder]
The capture window (cudaProfilerStart/Stop) covers only the second BFS from
`source`, after one warm BFS.
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
import paper_conf_ipps_gerak23_b200 as efg  # noqa: E402

src_v = int(sys.argv[1]) if len(sys.argv) > 1 else 5304443
reorder = (sys.argv[2] if len(sys.argv) > 2 else "degree") == "degree"
cfg = int(os.environ.get("EFG_PROF_CONFIG", "2"))
n, s, d = synth.config_edges(cfg)[:3]
flags = efg.EFG_DEFAULT_FLAGS | (efg.EFG_REORDER_DEGREE if reorder else 0)
stream = torch.cuda.Stream()
g = efg.Graph.build(n, s, d, stream=stream.cuda_stream, flags=flags)
del s, d
g.set_level_loop(True)
depth = torch.empty(n, dtype=torch.int32, device="cuda")
with torch.cuda.stream(stream):
    _, _, st = g.bfs(src_v, depth=depth, stats=True)
torch.cuda.synchronize()
print("levels", st["levels"], "edges", list(st["level_edges"]), file=sys.stderr)
torch.cuda.profiler.start()
with torch.cuda.stream(stream):
    g.bfs(src_v, depth=depth)
torch.cuda.synchronize()
torch.cuda.profiler.stop()
g.free()
