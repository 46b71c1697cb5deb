python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_ab.log 2>&1 || { tail -20 gpurun_out/build_ab.log; exit 1; }
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -3
timeout 900 python tools/ab_variant.py --config 3 --masks 1,3 --rounds 2 --levels 2>&1 | tail -1
timeout 600 python tools/ab_variant.py --config 2 --masks 1,3 --rounds 2 --levels 2>&1 | tail -1
