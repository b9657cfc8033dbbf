#!/bin/bash
# Panel QR grid size A/B: target rows per CTA (TRID_PANEL_ROWS), n = 8192 and n = 32768.
O=gpurun_out/r02pr; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for r in 64 128 256 32 64 128 256 32; do
  TRID_PANEL_ROWS=$r timeout 300 python bench.py --config n8192 --no-cpu-baseline --no-e2e --steps 5 --warmup 3 | sed "s/^/{\"rows\": $r, \"r\": /; s/\$/}/" >> $O/bench_n8192.jsonl 2>> $O/bench.err
done
for r in 64 128 64 128; do
  TRID_PANEL_ROWS=$r timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 2 --warmup 3 | sed "s/^/{\"rows\": $r, \"r\": /; s/\$/}/" >> $O/bench_n32768.jsonl 2>> $O/bench.err
done
ls -la $O
