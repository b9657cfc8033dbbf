#!/bin/bash
# Wide chase progress counters one 32-byte sector apart (default) vs packed (TRID_BC_FS=1): parity + interleaved A/B.
O=gpurun_out/r02fs; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_parity_large.py -q -x -m gpu -k "bulge" --timeout 300 > $O/pytest.log 2>&1
echo "pytest rc=$?" >> $O/pytest.log
timeout 900 python tools/bc_ab.py 32768 128 3 "fs8:" "fs1:TRID_BC_FS=1" > $O/ab.jsonl 2>&1
timeout 600 python tools/bc_ab.py 16384 128 3 "fs8:" "fs1:TRID_BC_FS=1" >> $O/ab.jsonl 2>&1
timeout 600 python tools/bc_ab.py 16384 256 3 "fs8:" "fs1:TRID_BC_FS=1" >> $O/ab.jsonl 2>&1
ls -la $O
