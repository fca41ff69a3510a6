#!/bin/bash
# One GPU iteration: parity tests, a band-group sweep of the bench, ncu on the flux kernels.
# usage (under gpurun): bash tools/gpu_iter.sh [tag] [bg-list] [ncu-bg]
cd $GRAFT_REPO_ROOT
TAG=${1:-iter}; BGS=${2:-"1 2 4 8"}; NBG=${3:-4}
OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > $OUT/pytest_gpu.log 2>&1
tail -3 $OUT/pytest_gpu.log
B="python bench.py --warmup 3 --no-cpu-baseline --no-e2e"
for bg in $BGS; do timeout 300 $B --steps 5 --band-group $bg >> $OUT/sweep.jsonl 2>>$OUT/sweep.err; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux -s 0 -c 1 -o $OUT/prof_flux $B --steps 1 --band-group $NBG > $OUT/ncu_full.log 2>&1
python - $OUT <<'PY'
import json,sys
for l in open(sys.argv[1]+'/sweep.jsonl'):
    d=json.loads(l); r=d['roofline']; p=d['phases_ms_per_step']
    print(d['band_group'], d['block_threads'], '%.3g upd/s'%d['value'], '%.2f ms'%d['ms_per_step'], 'int %.2f bnd %.2f newton %.2f'%(p['ms_flux_interior'],p['ms_flux_boundary'],p['ms_newton']), 'frac %.3f'%r['frac'])
PY
