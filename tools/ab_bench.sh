# A/B timing on one box: alternate the in-tree library and build/ab/libtrid_*.so (TRID_LIB_PATH), n = 32768 and 8192.
O=gpurun_out/${1:-ab}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1
for rep in 1 2; do
  for L in cur $(ls build/ab/ | sed 's/libtrid_//; s/.so//'); do
    if [ "$L" = cur ]; then unset TRID_LIB_PATH; else export TRID_LIB_PATH=$PWD/build/ab/libtrid_$L.so; fi
    timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > $O/b_${L}_${rep}.json 2> $O/b_${L}_${rep}.err
    timeout 600 python bench.py --config n8192 --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > $O/b8_${L}_${rep}.json 2> $O/b8_${L}_${rep}.err
  done
done
unset TRID_LIB_PATH
for f in $O/b*_*.json; do python -c "import json; d=json.load(open('$f')); print('$f', d['value'], d['t_bc_ms'], d['t_sbr_ms'])"; done > $O/summary.txt 2>&1
