#!/bin/bash
# Round-2 closing measurement, part B: headline bench (cpu baseline + e2e), reference arm, every BASELINE config,
# eigenvalues-only, the 8(f) rows, syr2k-vs-cuBLAS / cuSOLVER context, a launch list of one step, ncu --set full
# of the headline's dominant kernel (the first SYMM: 2nd ws_kernel launch) and of the syr2k.
O=gpurun_out/r02zb; mkdir -p $O
nvidia-smi > $O/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
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
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 5000 --csv --log-file $O/launches_n32768.csv \
  python bench.py --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > $O/launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ws_kernel --launch-skip 1 -c 1 \
  -o $O/symm_first python tools/prof_run.py --n 32768 --b 64 --k 1024 --nb 16 --stage sbr > $O/ncu_symm.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ws_kernel -c 1 \
  -o $O/syr2k python tools/syr2k_study.py --ns 32768 --ks 1024 --sytrd "" --reps 1 > $O/ncu_syr2k.log 2>&1
ls -la $O
# racecheck of the chase with the CTA-barrier hand-off (TRID_BC_OPT=0; bitwise-equal to the default per-warp
# __syncwarp + mbarrier hand-off, which racecheck does not model)
TRID_BC_OPT=0 TRID_PANEL_NOCOOP=1 timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_cases.py > $O/sanitize_racecheck_bcopt0.log 2>&1
echo "rc=$?" >> $O/sanitize_racecheck_bcopt0.log
