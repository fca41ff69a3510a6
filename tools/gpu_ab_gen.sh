#!/bin/bash
# A/B of generic-face kernel builds on C3t (bench + ncu) and the generic-kernel parity tests on the last lib.
cd $GRAFT_REPO_ROOT
TAG=$1; shift
OUT=gpurun_out/$TAG; mkdir -p $OUT
last=${@: -1}
BTE_DEBUG_SLOTS=1 BTE_LIB=$PWD/$last timeout 120 python -c "from paper_conf_ipps_heislersdms24_b200 import bte, inputs; s = bte.solver_from_config(inputs.make_config('C3t'), device=0)" 2>&1 | tail -2
BTE_LIB=$PWD/$last timeout 900 python -m pytest tests/test_gpu_n2.py -m gpu -q -x > $OUT/pytest.log 2>&1; tail -2 $OUT/pytest.log
for rep in 1 2; do
for lib in "$@"; do
  n=$(basename $lib .so)
  BTE_LIB=$PWD/$lib timeout 300 python bench.py --config C3t --warmup 3 --steps 20 --no-cpu-baseline --no-e2e > $OUT/${n}_$rep.json 2>$OUT/${n}_$rep.err
  python - $n $OUT/${n}_$rep.json <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[2]).read().strip().splitlines()[-1]); p=d['phases_ms_per_step']
    print(sys.argv[1], '| %.4g upd/s'%d['value'], '%.3f ms'%d['ms_per_step'], 'flux %.3f'%p['ms_flux_interior'], 'frac %.3f'%d['roofline']['frac'], d['clocks']['sm_mhz'], d['clocks']['reasons'])
except Exception as e: print(sys.argv[1], 'FAILED', e)
PY
done; done
for lib in "$@"; do
  n=$(basename $lib .so)
  BTE_LIB=$PWD/$lib timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux -s 3 -c 1 -o $OUT/prof_$n \
     python bench.py --config C3t --warmup 3 --steps 1 --no-cpu-baseline --no-e2e > $OUT/ncu_$n.log 2>&1
  ncu -i $OUT/prof_$n.ncu-rep --page raw --csv > $OUT/raw_$n.csv 2>/dev/null
  python tools/ncu_summary.py full $OUT/raw_$n.csv $OUT/sum_$n.json --config C3t; python -c "import json; k=json.load(open('$OUT/sum_$n.json'))['kernels'][0]; print(k.get('top_stalls'), k.get('instructions'), k.get('sm_pct_peak'))"
done
