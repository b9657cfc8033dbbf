#!/bin/bash
# Row-sharded MG corrections (virtual ranks on one device) + panel QR phase traces.
O=gpurun_out/r02mg; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_mg.py -q -x -m gpu --timeout 600 > $O/pytest_mg.log 2>&1; echo "rc=$?" >> $O/pytest_mg.log
for m in 4032 16320 32704; do
  TRID_PANEL_PAIR=0 timeout 300 python tools/panel_reg_trace.py $m 64 >> $O/panel_trace.log 2>&1
done
ls -la $O
