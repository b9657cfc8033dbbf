# BC hand-off options A/B (TRID_BC_OPT bitmask) on one box with tools/bc_bench.py, alternating
O=gpurun_out/${1:-bcopt}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for o in 2 4; do TRID_BC_OPT=$o timeout 300 python -m pytest tests/test_gpu_parity.py -x -q --timeout 120 -k "bulge" > $O/pytest_opt$o.log 2>&1; echo "rc=$?" >> $O/pytest_opt$o.log; done
for rep in 1 2; do
  for o in 0 1 2 4 7; do
    TRID_BC_OPT=$o timeout 300 python tools/bc_bench.py 32768 64 4 | sed "s/^{/{\"opt\": $o, /" >> $O/opt.jsonl 2>> $O/opt.err
    TRID_BC_OPT=$o timeout 300 python tools/bc_bench.py 8192 64 5 | sed "s/^{/{\"opt\": $o, /" >> $O/opt.jsonl 2>> $O/opt.err
  done
done
