#!/bin/bash
# Round-2 closing measurement (d: after the stacked U launch and the wide-chase changes): full -m gpu suite, smoke and the
# driver's plain-ncu smoke census, every BASELINE config's bench line, the reference arm, the 8(f) rows, the
# syr2k-vs-cuBLAS study, a full launch list of one headline step, ncu --set full of the SYMM (with folded
# corrections), the syr2k and the chase.
O=gpurun_out/r02d; mkdir -p $O
nvidia-smi > $O/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/smoke_launches_plain_ncu.csv \
  python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_ncu.log 2>&1; echo "rc=$?" >> $O/smoke_ncu.log
timeout 900 python bench.py > $O/bench_n32768.json 2> $O/bench_n32768.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference.json 2> $O/bench_reference.err
timeout 600 python bench.py --config n8192 --steps 5 --no-cpu-baseline > $O/bench_n8192.json 2> $O/bench_n8192.err
for c in n32768b128 n49152 n16384b32 n16384b64 n16384b128 n16384b256; do
  timeout 900 python bench.py --config $c --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > $O/bench_$c.json 2> $O/bench_$c.err
done
timeout 900 python bench.py --eig-only --no-cpu-baseline --no-e2e > $O/bench_n32768_eigonly.json 2> $O/bench_n32768_eigonly.err
timeout 900 python tools/bench_next.py --n 32768 --seed 3001 --rows f1,f3,evals > $O/next_n32768.jsonl 2>&1
timeout 900 python tools/bench_next.py --n 8192 --rows f1,f2,f3,evals > $O/next_n8192.jsonl 2>&1
timeout 1200 python tools/syr2k_study.py --ns 8192,32768,49152 --sytrd 8192,32768 > $O/syr2k_study.jsonl 2>&1
timeout 3000 python -m pytest tests -m gpu -q --timeout 900 -rA > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 7000 --csv --log-file $O/launches_n32768.csv \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > $O/launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ws_kernel --launch-skip 7 -c 1 \
  -o $O/prof_symm python tools/prof_run.py --n 32768 --b 64 --k 1024 --nb 16 --stage sbr > $O/ncu_symm.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ws_kernel -c 1 \
  -o $O/prof_syr2k python tools/syr2k_study.py --ns 32768 --ks 1024 --sytrd "" --reps 1 > $O/ncu_syr2k.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bc_v6 -c 1 \
  -o $O/prof_bc python tools/bc_ab.py 32768 64 1 "v6:" > $O/ncu_bc.log 2>&1
ls -la $O
