#!/bin/bash
O=gpurun_out/r02mb; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q --timeout 300 -k "bulge" > $O/pytest.log 2>&1
echo "pytest rc=$?" >> $O/pytest.log
timeout 900 python tools/bc_ab.py 32768 64 3 "default:TRID_BC_OPT=24" "mailbox:TRID_BC_OPT=88" > $O/bc_ab_n32768.txt 2>&1
timeout 600 python tools/bc_ab.py 8192 64 5 "default:TRID_BC_OPT=24" "mailbox:TRID_BC_OPT=88" > $O/bc_ab_n8192.txt 2>&1
timeout 600 python tools/bc_ab.py 16384 32 3 "default:TRID_BC_OPT=24" "mailbox:TRID_BC_OPT=88" > $O/bc_ab_n16384b32.txt 2>&1
ls -la $O
