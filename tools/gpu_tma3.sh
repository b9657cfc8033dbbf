#!/bin/bash
# Tensor-map TMA producer (TRID_WS_TMA=2) for the NT engine path: parity, syr2k and bench A/B vs the per-row bulk
# copies (1), ncu --set full of the syr2k with tensor maps.
O=gpurun_out/r02t3; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "syr2k or dbbr or two_stage or zy" --timeout 300 > $O/pytest.log 2>&1
echo "pytest rc=$?" >> $O/pytest.log
for t in 2 1 2 1; do
  TRID_WS_TMA=$t timeout 600 python tools/syr2k_study.py --ns 32768 --ks 1024 --sytrd "" | sed "s/^/{\"tma\": $t, \"r\": /; s/\$/}/" >> $O/syr2k.jsonl 2>&1
done
for t in 2 1 2 1; do
  TRID_WS_TMA=$t timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 3 | sed "s/^/{\"tma\": $t, \"r\": /; s/\$/}/" >> $O/bench.jsonl 2>> $O/bench.err
done
TRID_WS_TMA=2 timeout 600 ncu --set full --clock-control none --import-source on -k regex:ws_kernel -c 1 \
  -o $O/prof_syr2k python tools/syr2k_study.py --ns 32768 --ks 1024 --sytrd "" --reps 1 > $O/ncu.log 2>&1
ls -la $O
