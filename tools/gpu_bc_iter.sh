# BC iteration run (one gpurun call): parity suite, chase traces, bench lines, optional ncu source capture.
O=gpurun_out/${1:-r01m}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
timeout 300 python tools/bcw_trace.py 8192 64 1000 > $O/bcw6_trace_n8192.json 2>&1
timeout 300 python tools/bcw_trace.py 32768 64 20000 > $O/bcw6_trace_n32768_s20000.json 2>&1
timeout 300 python tools/bcw_trace.py 32768 64 2000 > $O/bcw6_trace_n32768_s2000.json 2>&1
timeout 900 python bench.py --no-cpu-baseline > $O/bench_n32768.json 2> $O/bench_n32768.err
timeout 600 python bench.py --config n8192 --steps 3 --no-cpu-baseline --no-e2e > $O/bench_n8192.json 2> $O/bench_n8192.err
if [ -n "$2" ]; then
  TRID_BC_FORCE=7 timeout 600 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $O/bench7_n32768.json 2> $O/bench7_n32768.err
  TRID_BC_FORCE=7 timeout 600 python bench.py --config n8192 --steps 3 --no-cpu-baseline --no-e2e > $O/bench7_n8192.json 2> $O/bench7_n8192.err
fi
