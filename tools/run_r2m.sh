python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python tools/ab_variant.py --config 3 --masks 43 --rounds 3 --levels 2>&1 | tail -1
timeout 900 python tools/ab_variant.py --config 2 --masks 43 --rounds 3 --levels 2>&1 | tail -1
EFG_FRONTIER_TRACE=1 EFG_PROF_CONFIG=3 timeout 900 python tools/prof_level.py 40483905 2>&1 | grep frontier-trace | head -5
