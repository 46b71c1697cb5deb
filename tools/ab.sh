#!/bin/bash
# same-box A/B of variants/NEW vs variants/OLD (alternating), plus the GPU tests of the in-tree build
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -1
bash tools/run_variants.sh NEW OLD NEW OLD
