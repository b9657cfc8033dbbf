O=gpurun_out/${1:-r01w}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
bash tools/gpu_bc_ab.sh $(basename $O)/bcab
bash tools/ab_bench.sh $(basename $O)/ab
