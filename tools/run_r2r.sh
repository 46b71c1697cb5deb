nvcc -gencode arch=compute_100a,code=sm_100a -o tools/ubench/mc_probe tools/ubench/mc_probe.cu -lcuda > gpurun_out/mc_build.log 2>&1 || { cat gpurun_out/mc_build.log; exit 1; }
timeout 120 tools/ubench/mc_probe 2>&1 | tee gpurun_out/mc_probe.txt
nvidia-smi topo -m 2>&1 | head -5
