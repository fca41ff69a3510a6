#!/bin/bash
# Experiment builds: bench + ncu of the first main flux launch per variant library.
# usage: bash tools/gpu_exp.sh TAG "BENCH-ARGS" lib1.so lib2.so ...
cd $GRAFT_REPO_ROOT
TAG=$1; A=$2; shift 2
OUT=gpurun_out/$TAG; mkdir -p $OUT
for lib in "$@"; do
  n=$(basename $lib .so)
  BTE_LIB=$PWD/$lib timeout 300 python bench.py --warmup 3 --steps 5 --no-cpu-baseline --no-e2e $A > $OUT/$n.json 2>$OUT/$n.err
  BTE_LIB=$PWD/$lib timeout 900 ncu --set full --clock-control none -k regex:flux -s 0 -c 1 -o $OUT/prof_$n \
     python bench.py --warmup 3 --steps 1 --no-cpu-baseline --no-e2e $A > $OUT/ncu_$n.log 2>&1
  python - $n $OUT/$n.json <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[2]).read().strip().splitlines()[-1]); p=d['phases_ms_per_step']
    print(sys.argv[1], '| %.3g upd/s'%d['value'], '%.2f ms'%d['ms_per_step'], 'flux %.2f'%p['ms_flux_interior'], 'frac %.3f'%d['roofline']['frac'])
except Exception as e: print(sys.argv[1], 'FAILED', e)
PY
done
