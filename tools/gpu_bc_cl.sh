# cluster-forwarding BC run: targeted parity first (bounded), then traces and benches per cluster size.
O=gpurun_out/${1:-r01q}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q --timeout 120 -k "cluster or variants" > $O/pytest_cl.log 2>&1; echo "rc=$?" >> $O/pytest_cl.log
if grep -q "rc=0" $O/pytest_cl.log; then
  for C in 2 4; do
    TRID_BC_FORCE=7 TRID_BC_CLUSTER=$C timeout 300 python tools/bcw_trace.py 8192 64 1000 > $O/bcw7c${C}_trace_n8192.json 2>&1
    TRID_BC_FORCE=7 TRID_BC_CLUSTER=$C timeout 600 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $O/bench7c${C}_n32768.json 2> $O/bench7c${C}_n32768.err
    TRID_BC_FORCE=7 TRID_BC_CLUSTER=$C timeout 600 python bench.py --config n8192 --steps 3 --no-cpu-baseline --no-e2e > $O/bench7c${C}_n8192.json 2> $O/bench7c${C}_n8192.err
  done
  TRID_BC_FORCE=7 timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 > $O/pytest_gpu_v7.log 2>&1; echo "rc=$?" >> $O/pytest_gpu_v7.log
fi
