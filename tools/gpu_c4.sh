#!/bin/bash
# C4 (web-shaped, ~7 B directed edges) measurements and full-size parity, one GPU.
TAG=${1:-c4}
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1 || { tail -20 $O/build_$TAG.log; exit 1; }
free -g | head -2
timeout 2400 python bench.py --config 4 --steps 6 --warmup 2 > $O/bench_${TAG}.json 2> $O/bench_${TAG}.err; echo "bench c4 rc=$?"; tail -c 2500 $O/bench_${TAG}.json
timeout 1800 python bench.py --config 4 --steps 6 --warmup 2 --permute --reorder none --no-sssp --no-alt --no-cpu-baseline > $O/bench_${TAG}_random.json 2> $O/bench_${TAG}_random.err; echo "bench c4 random rc=$?"; tail -c 600 $O/bench_${TAG}_random.json
timeout 1800 python tools/ab_variant.py --config 4 --masks 3,7 --rounds 1 --sources 4 --levels > $O/ab_${TAG}.json 2>&1; echo "ab rc=$?"; tail -1 $O/ab_${TAG}.json
timeout 3600 python tests/verify_full.py --config 4 --sources 2 --sssp > $O/verify_${TAG}.json 2> $O/verify_${TAG}.err; echo "verify rc=$?"; cat $O/verify_${TAG}.json
