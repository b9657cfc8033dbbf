#!/bin/bash
# SYMM mixed staging (tensor copies for the m-inner A tiles, cp.async for the rest; TRID_WS_TMA=2 default) vs
# all-cp.async (TRID_WS_TMA=1: the SYMM on cp.async, the syr2k on per-row bulk copies): parity + bench A/B.
O=gpurun_out/r02sm; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_large.py -q -x -m gpu -k "dbbr or zy or two_stage" --timeout 300 > $O/pytest.log 2>&1
echo "pytest rc=$?" >> $O/pytest.log
if grep -q "pytest rc=0" $O/pytest.log; then
  for t in 2 1 2 1; do
    TRID_WS_TMA=$t timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 3 | sed "s/^/{\"tma\": $t, \"r\": /; s/\$/}/" >> $O/bench.jsonl 2>> $O/bench.err
  done
  for t in 2 1; do
    TRID_WS_TMA=$t timeout 300 python bench.py --config n8192 --no-cpu-baseline --no-e2e --steps 5 --warmup 3 | sed "s/^/{\"tma\": $t, \"r\": /; s/\$/}/" >> $O/bench_n8192.jsonl 2>> $O/bench.err
  done
fi
ls -la $O
