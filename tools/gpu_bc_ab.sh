# low-noise chase A/B on one box: in-tree lib vs build/ab/libtrid_*.so, tools/bc_bench.py, alternating
O=gpurun_out/${1:-bcab}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
if [ -n "$2" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
fi
for rep in 1 2; do
  for L in cur $(ls build/ab/ | sed 's/libtrid_//; s/.so//'); do
    if [ "$L" = cur ]; then unset TRID_LIB_PATH; else export TRID_LIB_PATH=$PWD/build/ab/libtrid_$L.so; fi
    timeout 300 python tools/bc_bench.py 32768 64 5 >> $O/bc_ab.jsonl 2>> $O/bc_ab.err
    timeout 300 python tools/bc_bench.py 8192 64 7 >> $O/bc_ab.jsonl 2>> $O/bc_ab.err
  done
done
unset TRID_LIB_PATH
