python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
bash tools/build_variant.sh p1s4 "-DEFG_P1_SPARSE=4" > /dev/null 2>&1 &
bash tools/build_variant.sh p1s32 "-DEFG_P1_SPARSE=32" > /dev/null 2>&1 &
bash tools/build_variant.sh p1off "-DEFG_P1_SPARSE=1024" > /dev/null 2>&1 &
wait
for C in 2 3; do
for v in base p1s4 p1s32 p1off; do
  if [ $v = base ]; then L=$PWD/paper_conf_ipps_gerak23_b200/libefg.so; else L=$PWD/build/var_$v/libefg.so; fi
  echo -n "C$C $v: "; EFG_LIB=$L timeout 900 python tools/ab_variant.py --config $C --masks 43 --rounds 2 2>&1 | tail -1
done
done
EFG_PROF_CONFIG=3 timeout 1200 ncu --profile-from-start off --kernel-name regex:frontier --launch-skip 1 --launch-count 2 \
  --set full --import-source on --clock-control none -f -o gpurun_out/front_r2o python tools/prof_level.py 40483905 > gpurun_out/proff_r2o.log 2>&1; echo "ncu frontier rc=$?"
python tools/ncu_summary.py gpurun_out/front_r2o.ncu-rep "frontier_kernel, C3 level ends 1-2" > gpurun_out/front_r2o_summary.txt 2>&1
for L in 0 1; do python tools/ncu_lines.py gpurun_out/front_r2o.ncu-rep $L 50 > gpurun_out/front_lines_L$L.txt 2>&1; done
