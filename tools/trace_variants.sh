python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in K8 K4; do echo "== $v"; EFG_LIB=$PWD/variants/$v/libefg.so EFG_FRONTIER_TRACE=1 python tools/prof_level.py 2>&1 | grep trace | tail -8; done
