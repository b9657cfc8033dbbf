#!/bin/bash
# Final verification of the round-2 code: full -m gpu suite, smoke, headline and n = 8192 bench lines (with e2e).
O=gpurun_out/r02f; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 3000 python -m pytest tests -m gpu -q --timeout 900 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 900 python bench.py --no-cpu-baseline > $O/bench_n32768.json 2> $O/bench_n32768.err
timeout 600 python bench.py --config n8192 --steps 5 --no-cpu-baseline > $O/bench_n8192.json 2> $O/bench_n8192.err
ls -la $O
