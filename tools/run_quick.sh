#!/bin/bash
# quick GPU iteration: parity tests + bench on C2 (used via gpurun)
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -3
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --profile-levels 2>&1 | grep -E "L=[23] |metric|passed|failed|Error" | tail -14
