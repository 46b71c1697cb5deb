"""Turn an ncu metric capture of the expand launches of a bench run into
profiles/rNN_expand_traffic_<workload>.json (dram bytes per expand launch, and
the heaviest launch's bytes / duration / GB/s), which bench.py reports as
roofline.traffic and roofline.dram_heavy_launch.

On the GPU box:
  ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
      --clock-control none -k regex:expand --csv --log-file gpurun_out/expand_traffic.csv \
      python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-alt
Here:
  python tools/expand_traffic.py gpurun_out/expand_traffic.csv twitter_like degree [warm] \
      > profiles/r02_expand_traffic_twitter_like.json
(graph-mode launches are not profiled: ncu skips kernel nodes of graphs with
conditional nodes, so only the host-loop roofline pass appears)
"""
import csv
import json
import sys
from collections import defaultdict

path, workload, reorder = sys.argv[1:4]
warm = int(sys.argv[4]) if len(sys.argv) > 4 else 0  # leading launches to drop
rows = list(csv.reader(open(path)))
hdr = None
per = defaultdict(dict)
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        v = float(d["Metric Value"].replace(",", ""))
        unit = d.get("Metric Unit", "")
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1, "us": 1e3, "ms": 1e6}.get(unit, 1)
        per[d["ID"]][d["Metric Name"]] = v * scale
launches = [m for m in per.values() if "dram__bytes_read.sum" in m]
sel = launches[warm:] if len(launches) > warm else launches
tb = sum(m["dram__bytes_read.sum"] + m.get("dram__bytes_write.sum", 0) for m in sel)
tt = sum(m.get("gpu__time_duration.sum", 0) for m in sel)
hv = max(sel, key=lambda m: m["dram__bytes_read.sum"] + m.get("dram__bytes_write.sum", 0))
hb = hv["dram__bytes_read.sum"] + hv.get("dram__bytes_write.sum", 0)
ht = hv.get("gpu__time_duration.sum", 0)
out = {"workload": workload, "reorder": reorder, "launches": len(sel),
       "dram_bytes_per_launch": tb / max(len(sel), 1),
       "dram_gbps_cold": tb / max(tt, 1e-9),
       "heavy": {"dram_bytes": hb, "ns": ht, "gbps": hb / max(ht, 1e-9)},
       "source": f"ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum (cold cache, serialised) "
                 f"over {len(sel)} expand launches of bench.py; file {path}"}
print(json.dumps(out, indent=1))
