# ncu --set full of C3 levels 2-3 (base code) + per-line tables + raw l1tex metrics
bash tools/gpu_prof_c3.sh base
for L in 0 1; do python tools/ncu_lines.py gpurun_out/expand_base.ncu-rep $L 45 > gpurun_out/lines_base_L$L.txt 2>&1; done
ncu -i gpurun_out/expand_base.ncu-rep --page raw --csv > gpurun_out/raw_base.csv 2>&1
ls -la gpurun_out
