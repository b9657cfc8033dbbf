#!/bin/bash
# bench line for every BASELINE config (no cpu baseline / e2e): bash tools/gpu_configs.sh TAG [configs...]
TAG=${1:-r02}; shift
CFGS=${@:-"n8192 n32768 n32768b128 n49152 n16384b32 n16384b64 n16384b128 n16384b256"}
O=gpurun_out/$TAG; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for c in $CFGS; do
  timeout 900 python bench.py --config $c --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $O/bench_$c.json 2> $O/bench_$c.err
done
for c in $CFGS; do python -c "
import json,sys
try:
  d=json.load(open('$O/bench_$c.json'))
  print('$c', d['value'], 'sbr', d['t_sbr_ms'], 'bc', d['t_bc_ms'], d['stages_ms_per_step'], 'bcfrac', d['roofline_bc']['frac'], 'symm/syr2k frac', d['roofline']['frac'])
except Exception as e: print('$c', 'FAILED', e)
"; done > $O/summary.txt
