python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_q2.log 2>&1 || { tail -20 gpurun_out/build_q2.log; exit 1; }
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -4
timeout 600 python tools/ab_variant.py --config 2 --masks 3,7 --rounds 2 --levels 2>&1 | tail -1
timeout 900 python bench.py --config 2 --steps 4 --warmup 2 --host-resident --no-cpu-baseline --no-alt --no-pagerank --no-sssp 2>&1 | tail -1 | head -c 1500
