O=gpurun_out
python -c "import __graft_entry__ as g; g.build()" > $O/build_r2c.log 2>&1 || { tail -20 $O/build_r2c.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest_r2c.log 2>&1; tail -3 $O/pytest_r2c.log
timeout 900 python tools/ab_variant.py --config 3 --masks 3,11 --rounds 2 --levels 2>&1 | tail -1
timeout 600 python tools/ab_variant.py --config 2 --masks 3,11 --rounds 2 --levels 2>&1 | tail -1
bash tools/gpu_sanitize.sh
timeout 1800 python tests/verify_partitioned.py --scale 26 --world 8 --sources 2 > $O/verify_part26.json 2> $O/verify_part26.err; echo "verify_part rc=$?"; cat $O/verify_part26.json; tail -3 $O/verify_part26.err
