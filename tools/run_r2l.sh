python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
bash tools/build_variant.sh s2048r32 "-DEFG_STAGE_BYTES=2048 -DEFG_ROUND_WORDS=32" > /dev/null 2>&1 &
bash tools/build_variant.sh s2304r32 "-DEFG_STAGE_BYTES=2304 -DEFG_ROUND_WORDS=32" > /dev/null 2>&1 &
bash tools/build_variant.sh s2048 "-DEFG_STAGE_BYTES=2048" > /dev/null 2>&1 &
bash tools/build_variant.sh r32 "-DEFG_ROUND_WORDS=32" > /dev/null 2>&1 &
wait
ls build/var_*/libefg.so
for C in 3 2; do
for v in base s2048r32 s2304r32 s2048 r32; do
  if [ $v = base ]; then L=$PWD/paper_conf_ipps_gerak23_b200/libefg.so; else L=$PWD/build/var_$v/libefg.so; fi
  echo -n "C$C $v: "; EFG_LIB=$L timeout 900 python tools/ab_variant.py --config $C --masks 43 --rounds 2 --levels 2>&1 | tail -1
done
done
