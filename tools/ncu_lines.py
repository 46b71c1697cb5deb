"""Per-source-line instruction / stall / shared-wavefront totals of one kernel
launch from an .ncu-rep (needs -lineinfo and --import-source on).

usage: python tools/ncu_lines.py report.ncu-rep [launch_index] [top]
"""
import csv
import subprocess
import sys

rep = sys.argv[1]
li = int(sys.argv[2]) if len(sys.argv) > 2 else 0
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--launch-skip", str(li), "--launch-count", "1"], capture_output=True, text=True).stdout
def num(x):
    try:
        return int(float(x))
    except ValueError:
        return 0


rows = list(csv.reader(out.splitlines()))
hdr = None
agg = []
cur = None
for r in rows:
    if len(r) > 2 and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < len(hdr):
        continue
    d = dict(zip(hdr, r))
    if r[0]:  # a source line row (its metrics are the line totals)
        cur = [int(r[0]), r[1].strip()[:90], num(d["Instructions Executed"]),
               num(d["Warp Stall Sampling (All Samples)"]), num(d["L1 Wavefronts Shared"]),
               num(d["L1 Tag Requests Global"])]
        agg.append(cur)
tot = [sum(a[i] for a in agg) for i in range(2, 6)]
print(f"total: inst {tot[0]}  stall-samples {tot[1]}  smem-wavefronts {tot[2]}  global-tag-req {tot[3]}")
print(f"{'line':>5} {'inst%':>6} {'stall%':>6} {'smemwf%':>7} {'gtag%':>6}  source")
for a in sorted(agg, key=lambda a: -(a[2] / max(tot[0], 1) + a[3] / max(tot[1], 1)))[:top]:
    print(f"{a[0]:5d} {100*a[2]/max(tot[0],1):6.1f} {100*a[3]/max(tot[1],1):6.1f} "
          f"{100*a[4]/max(tot[2],1):7.1f} {100*a[5]/max(tot[3],1):6.1f}  {a[1]}")
