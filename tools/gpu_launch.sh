#!/bin/bash
O=gpurun_out/r02L; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file $O/launches.csv \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > $O/b.log 2>&1
ls -la $O
