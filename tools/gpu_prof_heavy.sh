#!/bin/bash
# ncu --set full of the heaviest C2 level: expand launch 3 and the plan launch before it.
TAG=${1:-cur}
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1 || { tail -20 $O/build_$TAG.log; exit 1; }
timeout 600 ncu --profile-from-start off --kernel-name regex:expand --launch-skip 3 --launch-count 1 \
  --set full --import-source on --clock-control none -f -o $O/expandL3_$TAG python tools/prof_level.py > $O/profL3_$TAG.log 2>&1; echo "ncu rc=$?"
timeout 600 ncu --profile-from-start off --kernel-name regex:plan --launch-skip 2 --launch-count 2 \
  --set full --import-source on --clock-control none -f -o $O/planL3_$TAG python tools/prof_level.py > $O/profP3_$TAG.log 2>&1; echo "ncu rc=$?"
python tools/ncu_summary.py $O/expandL3_$TAG.ncu-rep "expand L3 $TAG" > $O/expandL3_${TAG}_summary.txt 2>&1; cat $O/expandL3_${TAG}_summary.txt
python tools/ncu_summary.py $O/planL3_$TAG.ncu-rep "plan L2/L3 $TAG" > $O/planL3_${TAG}_summary.txt 2>&1; cat $O/planL3_${TAG}_summary.txt
