python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
EFG_DEBUG_LEVELS=1 EFG_FRONTIER_TRACE=1 EFG_PROF_CONFIG=3 timeout 900 python tools/prof_level.py 40483905 > gpurun_out/r2h_levels.log 2>&1
grep -E "efg-level|frontier-trace|levels" gpurun_out/r2h_levels.log | head -40
EFG_PROF_CONFIG=3 timeout 1200 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2h_launches.csv python tools/prof_level.py 40483905 > gpurun_out/r2h_ncu.log 2>&1
python - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/r2h_launches.csv')) if len(r)>10]
h=rows[0]; ki=h.index('Kernel Name'); mi=h.index('Metric Name'); vi=h.index('Metric Value'); ii=h.index('ID')
d={}
for r in rows[1:]:
    d.setdefault((int(r[ii]),r[ki][:40]),{})[r[mi]]=float(r[vi].replace(',',''))
for (i,k),m in sorted(d.items()):
    print(i,k,'%.1f us'%(m.get('gpu__time_duration.sum',0)/1e3),'rd %.0f MB'%(m.get('dram__bytes_read.sum',0)/1e6),'wr %.0f MB'%(m.get('dram__bytes_write.sum',0)/1e6))
PY
