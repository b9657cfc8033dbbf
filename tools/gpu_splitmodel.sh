#!/bin/bash
O=gpurun_out/r02m; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_large.py tests/test_gpu_backtransform.py -q --timeout 300 -k "zy or dbbr or two_stage or syr2k" > $O/pytest.log 2>&1
echo "pytest rc=$?" >> $O/pytest.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q --timeout 600 > $O/pytest_full.log 2>&1
echo "pytest rc=$?" >> $O/pytest_full.log
for f in 1 0 1 0; do
  TRID_SPLIT_MODEL=$f timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 3 | sed "s/^/{\"fold\": $f, \"r\": /; s/\$/}/" >> $O/bench.jsonl 2>> $O/bench.err
done
ls -la $O
