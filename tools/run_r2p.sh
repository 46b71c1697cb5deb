python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
bash tools/build_variant.sh gwold "-DEFG_GW_INTERLEAVE=0" > /dev/null 2>&1
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -2
for C in 3 2; do
for v in base gwold base gwold; do
  if [ $v = base ]; then L=$PWD/paper_conf_ipps_gerak23_b200/libefg.so; else L=$PWD/build/var_$v/libefg.so; fi
  echo -n "C$C $v: "; EFG_LIB=$L timeout 900 python tools/ab_variant.py --config $C --masks 43 --rounds 2 2>&1 | tail -1
done
done
EFG_FRONTIER_TRACE=1 EFG_PROF_CONFIG=3 timeout 900 python tools/prof_level.py 40483905 2>&1 | grep frontier-trace | head -5
