#!/bin/bash
O=gpurun_out/r02s2; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_large.py -q -x -k "zy or dbbr or two_stage" > $O/pytest.log 2>&1
echo "pytest rc=$?" >> $O/pytest.log
for w in new 8 new 8; do
  if [ $w = new ]; then unset TRID_SYMM_WAVES; else export TRID_SYMM_WAVES=$w; fi
  timeout 600 python bench.py --no-cpu-baseline --no-e2e --steps 3 --warmup 3 | sed "s/^/{\"symm\": \"$w\", \"r\": /; s/\$/}/" >> $O/bench.jsonl 2>> $O/bench.err
done
unset TRID_SYMM_WAVES
for m in 32704 28608 24512 16384 8192; do timeout 300 python tools/prof_symm.py --m $m --reps 6 >> $O/symm_new.jsonl 2>&1; done
export TRID_SYMM_WAVES=8
for m in 32704 28608 24512 16384 8192; do timeout 300 python tools/prof_symm.py --m $m --reps 6 >> $O/symm_old.jsonl 2>&1; done
ls -la $O
