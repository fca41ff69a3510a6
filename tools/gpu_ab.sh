#!/bin/bash
# A/B of library builds on the bench workloads: sustained bench lines, board
# power over 100 C4 steps, then one ncu --set full of the flux kernel each.
# usage: bash tools/gpu_ab.sh TAG "BENCH-ARGS" lib1.so lib2.so ...
cd $GRAFT_REPO_ROOT
TAG=$1; A=$2; shift 2
OUT=gpurun_out/$TAG; mkdir -p $OUT
for lib in "$@"; do
  n=$(basename $lib .so)
  for rep in 1 2; do
    BTE_LIB=$PWD/$lib timeout 300 python bench.py --warmup 3 --steps 20 --no-cpu-baseline --no-e2e $A > $OUT/${n}_$rep.json 2>$OUT/${n}_$rep.err
    python - "$n#$rep" $OUT/${n}_$rep.json <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[2]).read().strip().splitlines()[-1]); p=d['phases_ms_per_step']
    print(sys.argv[1], '| %.4g upd/s'%d['value'], '%.3f ms'%d['ms_per_step'], 'flux %.3f newton %.3f'%(p['ms_flux_interior'],p['ms_newton']), 'frac %.3f'%d['roofline']['frac'], d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'))
except Exception as e: print(sys.argv[1], 'FAILED', e)
PY
  done
  BTE_LIB=$PWD/$lib timeout 300 python tools/power_probe.py > $OUT/power_$n.txt 2>&1; echo "$n power: $(tail -2 $OUT/power_$n.txt | tr '\n' ' ')"
done
for lib in "$@"; do
  n=$(basename $lib .so)
  BTE_LIB=$PWD/$lib timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux -s 3 -c 1 -o $OUT/prof_$n \
     python bench.py --warmup 3 --steps 1 --no-cpu-baseline --no-e2e $A > $OUT/ncu_$n.log 2>&1
done
echo done
