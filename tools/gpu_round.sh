#!/bin/bash
# One GPU session: parity tests, smoke, bench lines, ncu launch list + traffic pass + full captures.
# usage (from the repo root, under gpurun):  bash tools/gpu_round.sh TAG [parts...]
TAG=${1:-r01}; shift
PARTS=${@:-"test bench launches traffic full"}
O=gpurun_out/$TAG
mkdir -p $O
nvidia-smi > $O/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
has() { [[ " $PARTS " == *" $1 "* ]]; }
if has test; then
  timeout 1500 python -m pytest tests -m gpu -q --timeout 300 > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
fi
if has bench; then
  timeout 900 python bench.py > $O/bench_n32768.json 2> $O/bench_n32768.err
  timeout 600 python bench.py --config n8192 --steps 5 --no-cpu-baseline > $O/bench_n8192.json 2> $O/bench_n8192.err
fi
CMD="python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
if has launches; then
  TRID_PANEL_NOCOOP=1 timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_n32768.csv $CMD > $O/launches.log 2>&1
fi
if has traffic; then
  TRID_PANEL_NOCOOP=1 timeout 1800 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum --clock-control none --csv --log-file $O/traffic_n32768.csv $CMD > $O/traffic.log 2>&1
fi
if has full; then
  P="python tools/prof_run.py --n 32768 --b 64 --k 1024 --nb 16"
  P8="python tools/prof_run.py --n 8192 --b 64 --k 1024 --nb 16"
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:bc_ -c 1 -o $O/prof_bc8192 $P8 > $O/prof_bc8192.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:ws_kernel -s 1 -c 1 -o $O/prof_symm $P > $O/prof_symm.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:ws_kernel<\(int\)128, \(int\)128' -c 1 -o $O/prof_syr2k $P > $O/prof_syr2k.log 2>&1
  TRID_PANEL_NOCOOP=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:panel_reg -s 5 -c 1 -o $O/prof_panel $P > $O/prof_panel.log 2>&1
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:bc_v6 -c 1 -o $O/prof_bc $P > $O/prof_bc.log 2>&1
fi
if has bctrace; then
  timeout 300 python tools/bcw_trace.py 8192 64 1000 > $O/bcw_trace_n8192.json 2>&1
  timeout 600 python tools/bcw_trace.py 32768 64 4000 > $O/bcw_trace_n32768.json 2>&1
  timeout 600 python tools/bcw_trace.py 32768 64 20000 > $O/bcw_trace_n32768_s20000.json 2>&1
fi
if has mgtest; then
  timeout 900 python -m pytest tests/test_gpu_mg.py -x -q --timeout 300 > $O/pytest_mg.log 2>&1; echo "rc=$?" >> $O/pytest_mg.log
fi
ls -la $O
