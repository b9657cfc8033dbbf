O=gpurun_out/${1:-r01v7}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for rep in 1 2; do
  for v in 6 7; do
    TRID_BC_FORCE=$v TRID_BC_CLUSTER=2 timeout 300 python tools/bc_bench.py 8192 64 5 >> $O/v7.jsonl 2>> $O/v7.err
    TRID_BC_FORCE=$v TRID_BC_CLUSTER=2 timeout 300 python tools/bc_bench.py 32768 64 3 >> $O/v7.jsonl 2>> $O/v7.err
  done
done
TRID_BC_FORCE=7 TRID_BC_CLUSTER=4 timeout 300 python tools/bc_bench.py 8192 64 5 >> $O/v7.jsonl 2>> $O/v7.err
