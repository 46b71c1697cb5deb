python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
bash tools/build_variant.sh ks4 "-DEFG_KS=4" > gpurun_out/b_ks4.log 2>&1 &
bash tools/build_variant.sh ks5 "-DEFG_KS=5" > /dev/null 2>&1 &
bash tools/build_variant.sh kb6 "-DEFG_KB=6" > /dev/null 2>&1 &
wait
grep -A2 "frontier_kernel" gpurun_out/b_ks4.log | grep -E "registers|spill" | head -2
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -2
for C in 3 2; do
for v in base ks4 ks5 kb6; do
  if [ $v = base ]; then L=$PWD/paper_conf_ipps_gerak23_b200/libefg.so; else L=$PWD/build/var_$v/libefg.so; fi
  echo -n "C$C $v: "; EFG_LIB=$L timeout 900 python tools/ab_variant.py --config $C --masks 43 --rounds 2 2>&1 | tail -1
done
done
