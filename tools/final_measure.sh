#!/bin/bash
# Round-end measurement set (via gpurun): tests, smoke, C2 bench + ncu, C3 and C4 bench lines.
bash tools/gpu_measure.sh fin
timeout 1500 python bench.py --config 3 --no-cpu-baseline --no-alt --no-pagerank --no-sssp > gpurun_out/bench_c3_fin.json 2> gpurun_out/bench_c3_fin.err; echo "c3 rc=$?"; tail -c 600 gpurun_out/bench_c3_fin.json
timeout 2400 python bench.py --config 4 --no-cpu-baseline --no-pagerank --no-sssp > gpurun_out/bench_c4_fin.json 2> gpurun_out/bench_c4_fin.err; echo "c4 rc=$?"; tail -c 600 gpurun_out/bench_c4_fin.json
