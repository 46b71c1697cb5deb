#!/bin/bash
# ncu launch list + expand dram traffic of bench.py (BFS only), TAG suffix
TAG=${1:-cur}; O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
NB="--steps 2 --warmup 1 --no-cpu-baseline --no-alt --no-pagerank --no-sssp"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
  python bench.py $NB > /dev/null 2>&1; echo "ncu list rc=$?"
python tools/launches.py $O/launches_$TAG.csv > $O/launches_${TAG}_summary.txt 2>&1; cat $O/launches_${TAG}_summary.txt
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none \
  -k regex:expand --csv --log-file $O/expand_traffic_$TAG.csv python bench.py $NB > /dev/null 2>&1; echo "ncu traffic rc=$?"
