O=gpurun_out/${1:-r01z}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for rep in 1 2; do
  for fs in 8 32 1; do
    TRID_BC_FS=$fs timeout 300 python tools/bc_bench.py 32768 64 4 | sed "s/^{/{\"fs\": $fs, /" >> $O/fs_ab.jsonl 2>> $O/fs_ab.err
    TRID_BC_FS=$fs timeout 300 python tools/bc_bench.py 8192 64 5 | sed "s/^{/{\"fs\": $fs, /" >> $O/fs_ab.jsonl 2>> $O/fs_ab.err
  done
done
timeout 300 python tools/bcw_trace.py 8192 64 1000 > $O/bcw6_trace_n8192.json 2>&1
timeout 300 python tools/bcw_trace.py 32768 64 2000 > $O/bcw6_trace_n32768_s2000.json 2>&1
timeout 300 python tools/bcw_trace.py 32768 64 20000 > $O/bcw6_trace_n32768_s20000.json 2>&1
