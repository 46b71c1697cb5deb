#!/bin/bash
# Round-2 final measurement set: tests, smoke, C3 default line + ncu evidence,
# on-disk EFG timing, C2 and C4 lines.  usage: tools/gpu_r2_final2.sh TAG
TAG=${1:-r02c}
O=gpurun_out; mkdir -p $O
bash tools/gpu_r2_final.sh $TAG
timeout 900 python tools/io_time.py 3 /tmp/efg_io_c3.efg > $O/io_$TAG.json 2> $O/io_$TAG.err; echo "io rc=$?"; cat $O/io_$TAG.json
timeout 1500 python bench.py --config 2 > $O/bench_c2_$TAG.json 2> $O/bench_c2_$TAG.err; echo "c2 rc=$?"; tail -c 600 $O/bench_c2_$TAG.json
timeout 3000 python bench.py --config 4 > $O/bench_c4_$TAG.json 2> $O/bench_c4_$TAG.err; echo "c4 rc=$?"; tail -c 600 $O/bench_c4_$TAG.json
