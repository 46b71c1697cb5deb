#!/bin/bash
# ncu --set full of the frontier_kernel launches after levels 1..3 of one C2 BFS
TAG=${1:-cur}
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1 || { tail -20 $O/build_$TAG.log; exit 1; }
timeout 600 ncu --profile-from-start off --kernel-name regex:frontier --launch-skip 2 --launch-count 3 \
  --set full --import-source on --clock-control none -f -o $O/front_$TAG python tools/prof_level.py > $O/proff_$TAG.log 2>&1; echo "ncu rc=$?"
python tools/ncu_summary.py $O/front_$TAG.ncu-rep "frontier L1-L3 $TAG" > $O/front_${TAG}_summary.txt 2>&1; cat $O/front_${TAG}_summary.txt
for i in 0 1 2; do python tools/ncu_lines.py $O/front_$TAG.ncu-rep $i 25; done
