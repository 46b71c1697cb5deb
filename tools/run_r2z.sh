python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
for D in 3 2; do
echo "div $D"
EFG_LPC_SKIP_DIV=$D timeout 2400 python tools/ab_variant.py --config 4 --masks 43,107 --rounds 2 --sources 10 2>&1 | tail -1
EFG_LPC_SKIP_DIV=$D timeout 1200 python tools/ab_variant.py --config 3 --masks 43,107 --rounds 2 --levels 2>&1 | tail -1
done
