python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 2400 python tools/ab_variant.py --config 4 --masks 43,107 --rounds 3 --sources 10 --levels 2>&1 | tail -1
