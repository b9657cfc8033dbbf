#!/bin/bash
O=gpurun_out/r02wt2; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 300 python tools/bcw_wide_trace.py 16384 128 2000 >> $O/trace.jsonl 2>&1
timeout 300 python tools/bcw_wide_trace.py 16384 128 200 >> $O/trace.jsonl 2>&1
timeout 300 python tools/bcw_wide_trace.py 16384 256 2000 >> $O/trace.jsonl 2>&1
