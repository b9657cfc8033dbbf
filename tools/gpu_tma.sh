#!/bin/bash
# TMA-staged engine A/B: parity + bitwise on/off, headline bench on/off, syr2k study on/off.
O=gpurun_out/r02t; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "syr2k or dbbr or two_stage or zy" > $O/pytest.log 2>&1
echo "pytest rc=$?" >> $O/pytest.log
for t in 1 0 1 0; do
  TRID_WS_TMA=$t timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 3 >> $O/bench_tma$t.json 2>> $O/bench.err
done
for t in 1 0; do
  TRID_WS_TMA=$t timeout 600 python tools/syr2k_study.py --ns 32768 --ks 256,512,1024,2048 --sytrd "" > $O/syr2k_tma$t.jsonl 2>&1
done
TRID_WS_TMA=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:ws_kernel -c 1 \
  -o $O/syr2k_tma1 python tools/syr2k_study.py --ns 32768 --ks 1024 --sytrd "" --reps 1 > $O/ncu.log 2>&1
TRID_WS_TMA=0 timeout 600 ncu --set full --clock-control none --import-source on -k regex:ws_kernel -c 1 \
  -o $O/syr2k_tma0 python tools/syr2k_study.py --ns 32768 --ks 1024 --sytrd "" --reps 1 >> $O/ncu.log 2>&1
ls -la $O
