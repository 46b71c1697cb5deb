python -c "import __graft_entry__ as g; g.build()" > gpurun_out/b.log 2>&1 || { tail gpurun_out/b.log; exit 1; }
EFG_FRONTIER_TRACE=1 python tools/prof_level.py 2>&1 | grep -E "trace|levels" | head -30
