O=gpurun_out/${1:-r01dir}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q --timeout 300 -k "bulge or sytrd or cluster" > $O/pytest_bc.log 2>&1; echo "rc=$?" >> $O/pytest_bc.log
if grep -q "rc=0" $O/pytest_bc.log; then
  bash tools/gpu_bc_ab.sh $(basename $O)/bcab
  timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
  timeout 300 python tools/bcw_trace.py 8192 64 1000 > $O/bcw6_trace_n8192.json 2>&1
  timeout 300 python tools/bcw_trace.py 32768 64 20000 > $O/bcw6_trace_n32768_s20000.json 2>&1
fi
