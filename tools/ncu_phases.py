"""Attribute an expand_kernel launch's instructions to its phases (source-line
ranges found by marker strings in efg_kernels.cu).  usage: ncu_phases.py rep idx elements"""
import csv
import subprocess
import sys

rep, li, E = sys.argv[1], sys.argv[2], float(sys.argv[3])
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--launch-skip", li, "--launch-count", "1"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr, agg = None, {}


def num(x):
    try:
        return float(x)
    except ValueError:
        return 0.0


for r in rows:
    if len(r) > 2 and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < len(hdr) or not r[0]:
        continue
    d = dict(zip(hdr, r))
    agg[int(r[0])] = (num(d["Instructions Executed"]), num(d["Thread Instructions Executed"]),
                      num(d["Warp Stall Sampling (All Samples)"]))
src = open("paper_conf_ipps_gerak23_b200/csrc/efg_kernels.cu").read().split("\n")


def find(pat):
    for i, l in enumerate(src):
        if pat in l:
            return i + 1
    return 10 ** 9


marks = [("producer", "auto produce = [&]"), ("slottable", "Batch cur, nxt;"), ("compaction", "uint32_t Er0 = 0;"),
         ("lanestart", "const uint32_t Er1 = run;"), ("decode", "auto decode = [&]"), ("visit", "auto visit = [&]"),
         ("loops", "// main loop: kU elements"), ("end", "atomicMax(&a.stats[xl].t1")]
pos = [(n, find(m)) for n, m in marks]
tot = sum(v[0] for v in agg.values())
tt = sum(v[1] for v in agg.values())
ts = sum(v[2] for v in agg.values())
print(f"total warp-inst {tot/1e6:.1f}M  thread-inst/elt {tt/E:.1f}  (elements {E:.0f})")
for (n, a), (_, b) in zip(pos[:-1], pos[1:]):
    s = sum(v[0] for l, v in agg.items() if a <= l < b)
    t = sum(v[1] for l, v in agg.items() if a <= l < b)
    st = sum(v[2] for l, v in agg.items() if a <= l < b)
    print(f"{n:12s} {100*s/tot:5.1f}% inst  thread-inst/elt {t/E:6.1f}  stall {100*st/max(ts,1):5.1f}%")
o = sum(v[1] for l, v in agg.items() if l < pos[0][1] or l >= pos[-1][1])
os_ = sum(v[2] for l, v in agg.items() if l < pos[0][1] or l >= pos[-1][1])
print(f"{'helpers':12s}       thread-inst/elt {o/E:6.1f}  stall {100*os_/max(ts,1):5.1f}%")
