O=gpurun_out/${1:-r01final2}; mkdir -p $O
nvidia-smi > $O/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 900 python bench.py > $O/bench_n32768.json 2> $O/bench_n32768.err
timeout 600 python bench.py --config n8192 --steps 5 --no-cpu-baseline > $O/bench_n8192.json 2> $O/bench_n8192.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $O/bench_reference.json 2> $O/bench_reference.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bc_v6 -c 1 -o $O/prof_bc python tools/prof_run.py --n 32768 --b 64 --k 1024 --nb 16 > $O/prof_bc.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:bc_v6 -c 1 -o $O/prof_bc8192 python tools/prof_run.py --n 8192 --b 64 --k 1024 --nb 16 > $O/prof_bc8192.log 2>&1
