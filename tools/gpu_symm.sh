#!/bin/bash
O=gpurun_out/r02s; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 300 python tools/prof_symm.py --m 32704 > $O/symm_time.json 2>&1
timeout 300 python tools/prof_symm.py --m 16384 >> $O/symm_time.json 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ws_kernel -c 1 \
  -o $O/symm python tools/prof_symm.py --m 32704 --reps 1 > $O/ncu.log 2>&1
ls -la $O
