#!/bin/bash
# Baseline of the C3 (twitter_like) headline config: box facts, per-level bench stats,
# ncu --set full of every expand launch of one C3 BFS.  usage: tools/gpu_c3_base.sh TAG
TAG=${1:-c3base}
O=gpurun_out; mkdir -p $O
{ nproc; free -g; lscpu | grep -E "Model name|Socket|Thread|Core|NUMA node\(s\)"; nvidia-smi --query-gpu=name,memory.total --format=csv; } > $O/box_$TAG.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1 || { tail -20 $O/build_$TAG.log; exit 1; }
timeout 900 python bench.py --config 3 --steps 5 --warmup 2 --no-cpu-baseline --no-alt --no-pagerank --no-sssp --profile-levels > $O/bench_$TAG.json 2> $O/bench_$TAG.err; echo "bench rc=$?"; tail -1 $O/bench_$TAG.json
EFG_PROF_CONFIG=3 timeout 1200 ncu --profile-from-start off --kernel-name regex:expand --launch-skip 0 --launch-count 6 \
  --set full --import-source on --clock-control none -f -o $O/expand_$TAG python tools/prof_level.py 40483905 > $O/prof_$TAG.log 2>&1; echo "ncu expand rc=$?"
python tools/ncu_summary.py $O/expand_$TAG.ncu-rep "expand_kernel, C3 all levels ($TAG)" > $O/expand_${TAG}_summary.txt 2>&1
grep -E "launch|gpu__time|dram__bytes_read|issue_active|warps_active" $O/expand_${TAG}_summary.txt | head -40
