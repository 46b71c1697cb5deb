"""On-disk EFG timing (efg_save / efg_load) on one BASELINE config: build from the
generator stream, save, load (host-only and onto the GPU), check equality.
  python tools/io_time.py [config] [path]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import synth  # noqa: E402
import paper_conf_ipps_gerak23_b200 as efg  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 3
path = sys.argv[2] if len(sys.argv) > 2 else "/tmp/efg_io_time.efg"
sg = synth.config_stream(cfg)
t = time.time()
g = efg.Graph.build_stream(sg.n, sg.m, sg.fn, sg.user, device=0, n_threads=os.cpu_count() or 1,
                           flags=efg.EFG_DEFAULT_FLAGS | efg.EFG_REORDER_DEGREE)
build_s = time.time() - t
t = time.time()
g.save(path)
save_s = time.time() - t
size = os.path.getsize(path)
os.system(f"sync; echo 3 > /proc/sys/vm/drop_caches 2>/dev/null")
t = time.time()
h = efg.Graph.load(path, device=0)
load_s = time.time() - t
src = int(synth.sources(sg.n, 1, seed=1000 + cfg)[0])
same = bool(np.array_equal(g.bfs(src), h.bfs(src)))
print(json.dumps({"config": cfg, "n": sg.n, "file_bytes": size, "build_s": round(build_s, 2),
                  "save_s": round(save_s, 2), "load_to_gpu_s": round(load_s, 2), "bfs_equal": same}))
os.remove(path)
