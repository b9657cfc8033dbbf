O=gpurun_out/${1:-r01x}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 > $O/pytest_gpu.log 2>&1; echo "rc=$?" >> $O/pytest_gpu.log
TRID_XUPD_SPLIT=0 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q --timeout 300 -k "dbbr or sytrd" > $O/pytest_noxs.log 2>&1; echo "rc=$?" >> $O/pytest_noxs.log
bash tools/ab_env.sh $(basename $O)/env "new:-" "skws:TRID_SKINNY_WS=1" "noxs:TRID_XUPD_SPLIT=0"
