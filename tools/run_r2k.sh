python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
bash tools/build_variant.sh bstat "-DEFG_BATCH_STATS=1" > gpurun_out/build_bstat.log 2>&1 || { tail gpurun_out/build_bstat.log; exit 1; }
EFG_LIB=$PWD/build/var_bstat/libefg.so EFG_DEBUG_LEVELS=1 EFG_PROF_CONFIG=3 timeout 900 python tools/prof_level.py 40483905 2>&1 | grep efg-level | head -6
EFG_LIB=$PWD/build/var_bstat/libefg.so EFG_DEBUG_LEVELS=1 EFG_PROF_CONFIG=2 timeout 900 python tools/prof_level.py 2>&1 | grep efg-level | head -9
