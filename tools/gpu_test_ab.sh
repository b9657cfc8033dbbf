# parity suite, then A/B bench (in-tree lib vs build/ab/*.so) on the same box
O=gpurun_out/${1:-r01t}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
bash tools/ab_bench.sh $(basename $O)/ab
timeout 300 python tools/bcw_trace.py 32768 64 2000 > $O/bcw6_trace_n32768_s2000.json 2>&1
timeout 300 python tools/bcw_trace.py 8192 64 1000 > $O/bcw6_trace_n8192.json 2>&1
