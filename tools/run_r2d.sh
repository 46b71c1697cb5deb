set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1200 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -3
timeout 900 python tools/ab_variant.py --config 3 --masks 11,27 --rounds 3 --levels 2>&1 | tail -3
timeout 600 python tools/ab_variant.py --config 2 --masks 11,27 --rounds 2 --levels 2>&1 | tail -1
