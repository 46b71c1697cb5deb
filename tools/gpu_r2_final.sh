#!/bin/bash
# Round-2 measurement set (via gpurun): GPU tests (all, incl. slow), smoke, the default
# bench line (C3), ncu launch list + expand dram traffic of the same bench command,
# ncu --set full of the C3 expand launches of levels 2-3.  usage: tools/gpu_r2_final.sh TAG
TAG=${1:-r02b}
O=gpurun_out; mkdir -p $O
{ nproc; free -g; lscpu | grep -E "Model name|Socket|Thread|Core"; nvidia-smi --query-gpu=name,memory.total,clocks.max.sm --format=csv; } > $O/box_$TAG.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1 || { tail -20 $O/build_$TAG.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest_$TAG.log 2>&1; tail -3 $O/pytest_$TAG.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_$TAG.log 2>&1; echo "smoke rc=$?"
timeout 1500 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err; echo "bench rc=$?"; tail -c 1500 $O/bench_$TAG.json
NB="--steps 2 --warmup 1 --no-cpu-baseline --no-alt --no-pagerank --no-sssp"
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
  python bench.py $NB > /dev/null 2>&1; echo "ncu list rc=$?"
python tools/launches.py $O/launches_$TAG.csv > $O/launches_${TAG}_summary.txt 2>&1; cat $O/launches_${TAG}_summary.txt
timeout 1200 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
  -k regex:expand --csv --log-file $O/expand_traffic_$TAG.csv python bench.py $NB > /dev/null 2>&1; echo "ncu traffic rc=$?"
python tools/expand_traffic.py $O/expand_traffic_$TAG.csv twitter_like degree > $O/traffic_$TAG.json; cat $O/traffic_$TAG.json
bash tools/gpu_prof_c3.sh $TAG
for L in 0 1; do python tools/ncu_lines.py $O/expand_$TAG.ncu-rep $L 60 > $O/lines_${TAG}_L$L.txt 2>&1; done
