#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over the C1-sized traversals:
# BFS (graph and host level loops, parents), decode, SSSP, PageRank, with
# the whole-graph, degree-relabelled and out-of-core builds.  Summaries -> gpurun_out/sanitize_<tool>.txt
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_san.log 2>&1 || { tail -20 $O/build_san.log; exit 1; }
for tool in memcheck racecheck synccheck; do
  timeout 1800 compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 \
    python tools/sanitize_target.py > $O/sanitize_$tool.txt 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|sanitize_target" $O/sanitize_$tool.txt | tail -3
done
