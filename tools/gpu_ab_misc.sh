#!/bin/bash
O=gpurun_out/r02x; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
run() { env $1 timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 3 | sed "s/^/{\"env\": \"$1\", \"r\": /; s/\$/}/" >> $O/bench.jsonl 2>> $O/bench.err; }
for rep in 1 2; do
  run "X=1"; run "TRID_ZY_WS=2"; run "TRID_WS_GROUP=4"; run "TRID_WS_GROUP=16"
done
ls -la $O
