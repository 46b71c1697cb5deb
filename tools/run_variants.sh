#!/bin/bash
# time each variants/<name>/libefg.so with bench.py (C2, short run)
for v in "$@"; do
  echo -n "$v: "
  EFG_LIB=$PWD/variants/$v/libefg.so timeout 300 python bench.py --steps 6 --warmup 3 --no-cpu-baseline --no-alt 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print('%.1f GTEPS  expand %.2f ms/launch-avg  roofline %.3f' % (d['value'], d['roofline']['expand_ms_total']/d['roofline']['expand_launches'], d['roofline']['frac']))
"
done
