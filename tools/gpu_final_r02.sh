#!/bin/bash
# Round-2 closing measurement, part A: full -m gpu suite, smoke, the driver's plain-ncu smoke census, sanitizers.
O=gpurun_out/r02z; mkdir -p $O
nvidia-smi > $O/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/smoke_launches_plain_ncu.csv \
  python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_ncu.log 2>&1; echo "rc=$?" >> $O/smoke_ncu.log
timeout 3000 python -m pytest tests -m gpu -q --timeout 900 -rA > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
for tool in racecheck synccheck; do
  TRID_PANEL_NOCOOP=1 timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_cases.py > $O/sanitize_$tool.log 2>&1
  echo "rc=$?" >> $O/sanitize_$tool.log
done
ls -la $O
