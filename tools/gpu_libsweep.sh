#!/bin/bash
# Bench-arg sweep for one library build. usage: bash tools/gpu_libsweep.sh TAG LIB "ARGS1" ...
cd $GRAFT_REPO_ROOT
TAG=$1; LIB=$2; shift 2
OUT=gpurun_out/$TAG; mkdir -p $OUT
for a in "$@"; do
  BTE_LIB=$PWD/$LIB timeout 300 python bench.py --warmup 3 --steps 5 --no-cpu-baseline --no-e2e $a > $OUT/one.json 2>>$OUT/sweep.err
  python - "$(basename $LIB) $a" $OUT/one.json >> $OUT/sweep.txt <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[2]).read().strip().splitlines()[-1]); r=d['roofline']; p=d['phases_ms_per_step']
    print(sys.argv[1], '| %.3g upd/s'%d['value'], '%.2f ms'%d['ms_per_step'], 'flux %.2f newton %.2f'%(p['ms_flux_interior'],p['ms_newton']), 'frac %.3f'%r['frac'], 'dch', d['dir_chunks'])
except Exception as e: print(sys.argv[1], 'FAILED', e)
PY
done
