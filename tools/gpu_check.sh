#!/bin/bash
# GPU pass (via gpurun): build, GPU tests, smoke, default bench line (C3), ncu traffic of the
# expand launches of the C3 roofline pass.  usage: tools/gpu_check.sh TAG [skip-tests] [skip-ncu]
TAG=${1:-cur}
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1 || { tail -20 $O/build_$TAG.log; exit 1; }
if [ "$2" != "skip-tests" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_$TAG.log 2>&1; tail -3 $O/pytest_$TAG.log
  timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_$TAG.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke_$TAG.log
fi
timeout 1200 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err; echo "bench rc=$?"; tail -c 3000 $O/bench_$TAG.json
if [ "$3" != "skip-ncu" ]; then
  NB="--steps 2 --warmup 1 --no-cpu-baseline --no-alt --no-pagerank --no-sssp"
  timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
    -k regex:expand --csv --log-file $O/expand_traffic_$TAG.csv python bench.py $NB > /dev/null 2>&1; echo "ncu traffic rc=$?"
  python tools/expand_traffic.py $O/expand_traffic_$TAG.csv twitter_like degree > $O/expand_traffic_$TAG.json; cat $O/expand_traffic_$TAG.json
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
    python bench.py $NB > /dev/null 2>&1; echo "ncu list rc=$?"
  python tools/launches.py $O/launches_$TAG.csv > $O/launches_${TAG}_summary.txt 2>&1; cat $O/launches_${TAG}_summary.txt
fi
