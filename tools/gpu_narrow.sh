#!/bin/bash
# 128x32 engine tiles for N <= 32 (b = 32 band): parity + A/B against the 128x64 tiles (TRID_WS_NARROW=0).
O=gpurun_out/r02nw; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_large.py tests/test_gpu_fullsize.py tests/test_gpu_backtransform.py -q -x -m gpu --timeout 600 > $O/pytest.log 2>&1
echo "pytest rc=$?" >> $O/pytest.log
for nw in 1 0 1 0; do
  TRID_WS_NARROW=$nw timeout 600 python bench.py --config n16384b32 --no-cpu-baseline --no-e2e --steps 2 --warmup 3 | sed "s/^/{\"narrow\": $nw, \"r\": /; s/\$/}/" >> $O/bench.jsonl 2>> $O/bench.err
done
ls -la $O
