"""Condense an .ncu-rep into a committed text summary (profiles/).

usage: python tools/ncu_summary.py report.ncu-rep [title] > profiles/<name>.txt
Prints per launch the duration, DRAM traffic, L2 sectors, issue / warp / L1 / L2
utilisation, then the stall-reason totals and the instruction mix of the
heaviest launch (from the SASS source page, needs -lineinfo).
"""
import collections
import csv
import subprocess
import sys

rep = sys.argv[1]
title = sys.argv[2] if len(sys.argv) > 2 else rep
print(f"# ncu summary: {title}\n# report: {rep}")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(raw.splitlines()))
hdr, units = r[0], r[1]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sectors.sum",
        "sm__inst_executed.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "l1tex__throughput.avg.pct_of_peak_sustained_active",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct", "launch__grid_size", "launch__block_size",
        "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic"]
for row in r[2:]:
    d = dict(zip(hdr, row))
    print(f"\n## launch {d['ID']}: {d['Kernel Name'][:90]}")
    for w in want:
        if w in d:
            print(f"  {w:58s} {d[w]:>16s} {units[hdr.index(w)]}")

src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(src.splitlines()))
kern, cur, shdr = [], None, None
for x in rows:
    if x and x[0] == "Kernel Name":
        cur = []
        kern.append(cur)
        continue
    if x and x[0] == "Address":
        shdr = x
        continue
    if cur is not None and x:
        cur.append(x)
if kern and shdr:
    H = {h: i for i, h in enumerate(shdr)}
    k = max(kern, key=lambda k: sum(int(x[H["Instructions Executed"]] or 0) for x in k))
    tot = sum(int(x[H["Instructions Executed"]] or 0) for x in k)
    stalls = [h for h in shdr if h.startswith("stall_") and "Not Issued" not in h]
    agg = {s: sum(int(x[H[s]] or 0) for x in k) for s in stalls}
    ts = sum(agg.values()) or 1
    print(f"\n## heaviest kernel: {tot} warp instructions executed")
    print("## stall reasons (share of samples):")
    for s, v in sorted(agg.items(), key=lambda t: -t[1])[:10]:
        print(f"  {s:28s} {v / ts:6.1%}")
    ops = collections.Counter()
    for x in k:
        t = x[1].strip().split()
        if not t:
            continue
        op = t[1] if t[0].startswith("@") and len(t) > 1 else t[0]
        ops[op.split(".")[0]] += int(x[H["Instructions Executed"]] or 0)
    print("## instruction mix (top 16):")
    for op, c in ops.most_common(16):
        print(f"  {op:12s} {c / tot:6.1%}")
