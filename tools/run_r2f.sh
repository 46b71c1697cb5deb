python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
bash tools/build_variant.sh lwin "-DEFG_LWIN=1" > gpurun_out/build_lwin.log 2>&1 || { tail gpurun_out/build_lwin.log; exit 1; }
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,temperature.gpu,power.draw --format=csv
timeout 600 python -m pytest tests/test_gpu_bfs.py -k "variants" -x -q 2>&1 | tail -3
EFG_LIB=$PWD/build/var_lwin/libefg.so timeout 600 python -m pytest tests/test_gpu_bfs.py -k "variants" -x -q 2>&1 | tail -3
for i in 1 2; do
timeout 900 python tools/ab_variant.py --config 3 --masks 11,43 --rounds 2 --levels 2>&1 | tail -1
EFG_LIB=$PWD/build/var_lwin/libefg.so timeout 900 python tools/ab_variant.py --config 3 --masks 43,107 --rounds 2 --levels 2>&1 | tail -1
done
