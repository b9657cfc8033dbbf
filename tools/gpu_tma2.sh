#!/bin/bash
# Engine epilogue / Cin prefetch / grouped order A/B.
O=gpurun_out/r02t2; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "syr2k or dbbr or two_stage or zy" > $O/pytest.log 2>&1
echo "pytest rc=$?" >> $O/pytest.log
for cfg in "1 8" "1 1" "2 8" "0 8" "0 1"; do
  set -- $cfg
  TRID_WS_TMA=$1 TRID_WS_GROUP=$2 timeout 600 python tools/syr2k_study.py --ns 32768 --ks 1024 --sytrd "" | sed "s/^/{\"tma\": $1, \"group\": $2, \"r\": /; s/\$/}/" >> $O/syr2k.jsonl 2>&1
done
for cfg in "1 8" "1 1" "1 8" "1 1"; do
  set -- $cfg
  TRID_WS_TMA=$1 TRID_WS_GROUP=$2 timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 3 | sed "s/^/{\"tma\": $1, \"group\": $2, \"r\": /; s/\$/}/" >> $O/bench.jsonl 2>> $O/bench.err
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ws_kernel -c 1 \
  -o $O/syr2k_new python tools/syr2k_study.py --ns 32768 --ks 1024 --sytrd "" --reps 1 > $O/ncu.log 2>&1
ls -la $O
