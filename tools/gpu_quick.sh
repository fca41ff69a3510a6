#!/bin/bash
# Quick check: smoke, solve-phase timing of C4 / C3 / C3t, a parity subset.
cd $GRAFT_REPO_ROOT
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
for spec in "C4 20" "C3 50" "C3t 20"; do
  set -- $spec
  timeout 600 python bench.py --config $1 --steps $2 --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['phases_ms_per_step']; print('$1 %.4g upd/s flux %.3f newton %.4f frac %.3f it %s' % (d['value'], p['ms_flux_interior'], p['ms_newton'], d['roofline']['frac'], d.get('newton_iter_max')))"
done
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_r2.py tests/test_gpu_n1.py tests/test_gpu_box.py -m gpu -q -x 2>&1 | tail -2
