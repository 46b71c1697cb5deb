python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
nvcc -gencode arch=compute_100a,code=sm_100a -o tools/ubench/mc_probe tools/ubench/mc_probe.cu -lcuda > gpurun_out/mc_build.log 2>&1 || { cat gpurun_out/mc_build.log; exit 1; }
timeout 120 tools/ubench/mc_probe 2>&1 | tee gpurun_out/mc_probe.txt
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --tb=short 2>&1 | tail -15
