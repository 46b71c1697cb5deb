#!/bin/bash
# One GPU measurement pass (run via gpurun): parity tests, bench line, ncu launch list,
# ncu --set full capture of the two heaviest expand launches of one C2 BFS.
# usage: tools/gpu_measure.sh TAG
TAG=${1:-cur}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1 || { tail -20 $O/build_$TAG.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_$TAG.log 2>&1; tail -3 $O/pytest_$TAG.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_$TAG.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err; echo "bench rc=$?"; tail -1 $O/bench_$TAG.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-alt > $O/launches_bench_$TAG.log 2>&1; echo "ncu list rc=$?"
python tools/launches.py $O/launches_$TAG.csv > $O/launches_${TAG}_summary.txt 2>&1; cat $O/launches_${TAG}_summary.txt
timeout 900 ncu --profile-from-start off --kernel-name regex:expand --launch-skip 1 --launch-count 2 \
  --set full --import-source on --clock-control none -f -o $O/expand_$TAG python tools/prof_level.py > $O/prof_$TAG.log 2>&1; echo "ncu full rc=$?"
python tools/ncu_summary.py $O/expand_$TAG.ncu-rep "expand $TAG" > $O/expand_${TAG}_summary.txt 2>&1; head -40 $O/expand_${TAG}_summary.txt
