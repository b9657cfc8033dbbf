#!/bin/bash
# Round-2 final numbers after the SYMM mixed staging: headline (cpu baseline + e2e), the other configs, the
# eigenvalues-only line, ncu --set full of the SYMM (panel 1, with corrections), the full -m gpu suite.
O=gpurun_out/r02e; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python bench.py > $O/bench_n32768.json 2> $O/bench_n32768.err
timeout 600 python bench.py --config n8192 --steps 5 --no-cpu-baseline > $O/bench_n8192.json 2> $O/bench_n8192.err
for c in n32768b128 n49152 n16384b32 n16384b64 n16384b128 n16384b256; do
  timeout 900 python bench.py --config $c --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $O/bench_$c.json 2> $O/bench_$c.err
done
timeout 900 python bench.py --eig-only --no-cpu-baseline --no-e2e > $O/bench_n32768_eigonly.json 2> $O/bench_n32768_eigonly.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ws_kernel --launch-skip 6 -c 1 \
  -o $O/prof_symm python tools/prof_run.py --n 32768 --b 64 --k 1024 --nb 16 --stage sbr > $O/ncu_symm.log 2>&1
timeout 2200 python -m pytest tests/ -q -m gpu > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
ls -la $O
