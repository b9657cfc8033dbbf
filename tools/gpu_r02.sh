#!/bin/bash
# Round-2 GPU session driver: bash tools/gpu_r02.sh TAG part...   (parts: test smoke bench bench8k b128 san full launches)
TAG=${1:-r02}; shift
PARTS=" $* "
O=gpurun_out/$TAG
mkdir -p $O
nvidia-smi > $O/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
has() { [[ "$PARTS" == *" $1 "* ]]; }
if has test; then
  timeout 2400 python -m pytest tests -m gpu -q --timeout 900 -x -rA > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
fi
if has testfast; then
  timeout 1800 python -m pytest tests -m gpu -q --timeout 600 -rA --deselect tests/test_gpu_fullsize.py > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
fi
if has smoke; then
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
fi
if has san; then
  for tool in racecheck synccheck memcheck; do
    TRID_PANEL_NOCOOP=1 timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_cases.py > $O/sanitize_$tool.log 2>&1
    echo "rc=$?" >> $O/sanitize_$tool.log
  done
fi
if has bench; then
  timeout 900 python bench.py > $O/bench_n32768.json 2> $O/bench_n32768.err
fi
if has bench8k; then
  timeout 600 python bench.py --config n8192 --steps 5 --no-cpu-baseline > $O/bench_n8192.json 2> $O/bench_n8192.err
fi
if has b128; then
  timeout 900 python bench.py --config n32768b128 --no-cpu-baseline --no-e2e > $O/bench_n32768b128.json 2> $O/bench_n32768b128.err
fi
if has ncusmoke; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/smoke_launches.csv python -c "import __graft_entry__ as g; g.smoke()" > $O/ncusmoke.log 2>&1
  echo "rc=$?" >> $O/ncusmoke.log
fi
if has launches; then
  timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_n32768.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > $O/launches.log 2>&1
  echo "rc=$?" >> $O/launches.log
fi
ls -la $O
