#!/bin/bash
# Quick pass: GPU suite + bench lines of C4 / C3 / C3t / C4 rate law (phase times).
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-s2}; mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q -x --timeout 1500 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -5 $OUT/pytest_gpu.log
for spec in "C4 20" "C3 50" "C3t 20"; do
  set -- $spec
  timeout 600 python bench.py --config $1 --steps $2 --no-cpu-baseline --no-e2e > $OUT/bench_$1.json 2> $OUT/bench_$1.err
  python - $1 $OUT/bench_$1.json <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[2]).read().strip().splitlines()[-1]); p=d['phases_ms_per_step']
    print(sys.argv[1], '| %.4g upd/s'%d['value'], '%.3f ms'%d['ms_per_step'], 'flux %.3f'%p['ms_flux_interior'], 'newton %.4f'%p['ms_newton'], 'frac %.3f'%d['roofline']['frac'], 'it', d.get('newton_iter_max'), d['clocks']['sm_mhz'], d['clocks']['reasons'])
except Exception as e: print(sys.argv[1], 'FAILED', e)
PY
done
timeout 600 python bench.py --rate-law --steps 20 --no-cpu-baseline --no-e2e > $OUT/bench_C4_ratelaw.json 2> $OUT/bench_C4_ratelaw.err
tail -1 $OUT/bench_C4_ratelaw.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C4 law', d['value'], d['phases_ms_per_step'], d.get('newton_iter_max'))"
