#!/bin/bash
# quick GPU iteration: build, parity tests + bench on C2 (used via gpurun)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_quick.log 2>&1 || { tail -20 gpurun_out/build_quick.log; exit 1; }
timeout 900 python -m pytest tests -m "gpu" -x -q 2>&1 | tail -15
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --profile-levels 2>&1 | tail -30
