python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
EFG_PROF_CONFIG=3 timeout 1200 ncu --profile-from-start off --kernel-name regex:frontier --launch-skip 3 --launch-count 1 \
  --set full --import-source on --clock-control none -f -o gpurun_out/front_l2end python tools/prof_level.py 40483905 > gpurun_out/proff_l2end.log 2>&1; echo "ncu frontier rc=$?"
python tools/ncu_summary.py gpurun_out/front_l2end.ncu-rep "frontier_kernel, C3 level-2 end" > gpurun_out/front_l2end_summary.txt 2>&1
python tools/ncu_lines.py gpurun_out/front_l2end.ncu-rep 0 60 > gpurun_out/front_l2end_lines.txt 2>&1
cat gpurun_out/front_l2end_summary.txt | head -45; head -45 gpurun_out/front_l2end_lines.txt
