#!/bin/bash
# Full measurement session: headline bench (cpu baseline + e2e), every BASELINE config, the 8(f) rows.
TAG=${1:-r02}; O=gpurun_out/$TAG; mkdir -p $O
nvidia-smi > $O/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python bench.py > $O/bench_n32768.json 2> $O/bench_n32768.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > $O/bench_reference.json 2> $O/bench_reference.err
bash tools/gpu_configs.sh $TAG n8192 n32768b128 n49152 n16384b32 n16384b64 n16384b128 n16384b256
timeout 900 python bench.py --eig-only --no-cpu-baseline --no-e2e > $O/bench_n32768_eigonly.json 2> $O/bench_n32768_eigonly.err
timeout 900 python tools/bench_next.py --n 32768 --seed 3001 --rows f1,f3,evals > $O/next_n32768.jsonl 2>&1
timeout 900 python tools/bench_next.py --n 8192 --rows f1,f2,f3,evals > $O/next_n8192.jsonl 2>&1
ls -la $O
