python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_peer_ipc.py -x -q 2>&1 | tail -2
for C in 1 2; do
EFG_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 2951$C bench.py --gpus 2 --config $C --steps 3 --warmup 3 > gpurun_out/bench_2r_c$C.json 2> gpurun_out/bench_2r_c$C.err; echo "rc=$?"; tail -1 gpurun_out/bench_2r_c$C.json; tail -3 gpurun_out/bench_2r_c$C.err
done
