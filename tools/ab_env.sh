# A/B of env-selected variants of the in-tree library on one box (full bench, n = 32768), alternating.
# usage: bash tools/ab_env.sh OUTDIR "NAME1:ENV1=V1" "NAME2:ENV2=V2" ...   (ENV "-" = none)
O=gpurun_out/$1; shift; mkdir -p $O
for rep in 1 2; do
  for spec in "$@"; do
    name=${spec%%:*}; env=${spec#*:}
    if [ "$env" = "-" ]; then env=""; fi
    env $env timeout 600 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > $O/b_${name}_${rep}.json 2> $O/b_${name}_${rep}.err
  done
done
for f in $O/b_*.json; do python -c "import json; d=json.load(open('$f')); print('$f', d['value'], d['t_bc_ms'], d['t_sbr_ms'], d['stages_ms_per_step'])"; done > $O/summary.txt 2>&1
