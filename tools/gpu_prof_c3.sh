#!/bin/bash
# ncu --set full of the expand launches of one C3 BFS (host level loop), plus plan statistics.
# usage: tools/gpu_prof_c3.sh TAG [source]
TAG=${1:-cur}; SRC=${2:-40483905}
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1 || { tail -20 $O/build_$TAG.log; exit 1; }
EFG_DEBUG_LEVELS=1 EFG_PROF_CONFIG=3 timeout 1200 ncu --profile-from-start off --kernel-name regex:expand --launch-skip 2 --launch-count 2 \
  --set full --import-source on --clock-control none -f -o $O/expand_$TAG python tools/prof_level.py $SRC > $O/prof_$TAG.log 2>&1; echo "ncu expand rc=$?"
grep efg-level $O/prof_$TAG.log | head -12
python tools/ncu_summary.py $O/expand_$TAG.ncu-rep "expand_kernel, C3 levels 2-3 ($TAG)" > $O/expand_${TAG}_summary.txt 2>&1
grep -E "launch|gpu__time|dram__bytes_read|issue_active|warps_active|warp instr" $O/expand_${TAG}_summary.txt | head -40
