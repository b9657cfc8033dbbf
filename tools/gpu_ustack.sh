#!/bin/bash
# Stacked U = -[Z_<^T W; Y_<^T W] (one launch) vs two launches (TRID_ZY_USTACK=0): parity + bench A/B.
O=gpurun_out/r02us; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_large.py tests/test_gpu_mg.py -q -x -m gpu -k "dbbr or zy or two_stage or mg" --timeout 300 > $O/pytest.log 2>&1
echo "pytest rc=$?" >> $O/pytest.log
for u in 1 0 1 0; do
  TRID_ZY_USTACK=$u timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 3 | sed "s/^/{\"ustack\": $u, \"r\": /; s/\$/}/" >> $O/bench.jsonl 2>> $O/bench.err
done
for u in 1 0; do
  TRID_ZY_USTACK=$u timeout 300 python bench.py --config n8192 --no-cpu-baseline --no-e2e --steps 5 --warmup 3 | sed "s/^/{\"ustack\": $u, \"r\": /; s/\$/}/" >> $O/bench_n8192.jsonl 2>> $O/bench.err
done
ls -la $O
