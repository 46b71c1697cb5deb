#!/bin/bash
# One GPU measurement pass (run via gpurun): parity tests, bench line, ncu launch list,
# expand dram traffic, ncu --set full of the heaviest expand and frontier launches of one C2 BFS.
# usage: tools/gpu_measure.sh TAG [skip-tests]
TAG=${1:-cur}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1 || { tail -20 $O/build_$TAG.log; exit 1; }
if [ "$2" != "skip-tests" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_$TAG.log 2>&1; tail -3 $O/pytest_$TAG.log
  timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_$TAG.log 2>&1; echo "smoke rc=$?"
fi
timeout 900 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err; echo "bench rc=$?"; tail -1 $O/bench_$TAG.json
NB="--steps 2 --warmup 1 --no-cpu-baseline --no-alt --no-pagerank --no-sssp"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
  python bench.py $NB > /dev/null 2>&1; echo "ncu list rc=$?"
python tools/launches.py $O/launches_$TAG.csv > $O/launches_${TAG}_summary.txt 2>&1; cat $O/launches_${TAG}_summary.txt
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
  -k regex:expand --csv --log-file $O/expand_traffic_$TAG.csv python bench.py $NB > /dev/null 2>&1; echo "ncu traffic rc=$?"
timeout 900 ncu --profile-from-start off --kernel-name regex:expand --launch-skip 2 --launch-count 2 \
  --set full --import-source on --clock-control none -f -o $O/expand_$TAG python tools/prof_level.py > $O/prof_$TAG.log 2>&1; echo "ncu expand rc=$?"
timeout 900 ncu --profile-from-start off --kernel-name regex:frontier --launch-skip 2 --launch-count 3 \
  --set full --import-source on --clock-control none -f -o $O/front_$TAG python tools/prof_level.py > $O/proff_$TAG.log 2>&1; echo "ncu frontier rc=$?"
python tools/ncu_summary.py $O/expand_$TAG.ncu-rep "expand_kernel, C2 levels 2-3 ($TAG)" > $O/expand_${TAG}_summary.txt 2>&1
python tools/ncu_summary.py $O/front_$TAG.ncu-rep "frontier_kernel, C2 level ends 1-3 ($TAG)" > $O/front_${TAG}_summary.txt 2>&1
grep -E "launch|gpu__time|dram__bytes|issue_active" $O/expand_${TAG}_summary.txt | head -20
