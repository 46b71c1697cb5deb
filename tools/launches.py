"""Summarise an ncu --metrics gpu__time_duration.sum launch list (csv)."""
import csv
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
hdr = None
out = []
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        out.append((d["Kernel Name"].split("(")[0].split("::")[-1], float(d["Metric Value"])))
tail = int(sys.argv[2]) if len(sys.argv) > 2 else 0
for i, (k, v) in enumerate(out[-tail:] if tail else []):
    print(i, k, v)
agg = defaultdict(lambda: [0, 0.0])
for k, v in out:
    agg[k][0] += 1
    agg[k][1] += v
tot = sum(v for _, v in agg.values())
for k, (c, v) in sorted(agg.items(), key=lambda t: -t[1][1]):
    print(f"{k:40s} launches={c:5d} total_ns={v:12.0f} share={v / tot:6.1%}")
