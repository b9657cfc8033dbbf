#!/bin/bash
# Wide chase with register-cached step vectors and direct column stores: parity, traces, config benches.
O=gpurun_out/r02w7; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_large.py -q -x -m gpu -k "bulge or two_stage" --timeout 300 > $O/pytest.log 2>&1
echo "pytest rc=$?" >> $O/pytest.log
if grep -q "pytest rc=0" $O/pytest.log; then
  timeout 300 python tools/bcw_wide_trace.py 16384 128 2000 >> $O/trace.jsonl 2>&1
  timeout 300 python tools/bcw_wide_trace.py 16384 256 2000 >> $O/trace.jsonl 2>&1
  for c in n32768b128 n16384b128 n16384b256; do
    timeout 900 python bench.py --config $c --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $O/bench_$c.json 2> $O/bench_$c.err
  done
fi
ls -la $O
