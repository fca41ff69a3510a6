#!/bin/bash
# Temperature-solve variants on C4 / C3 (BTE_NEWTON), ms per step of the solve phase.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-nab}; mkdir -p $OUT
for c in C4 C3; do for m in auto thread lanes4 lanes8 lanes16 warp; do
  if [ $m = auto ]; then E=""; else E="BTE_NEWTON=$m"; fi
  env $E timeout 300 python bench.py --config $c --steps 20 --no-cpu-baseline --no-e2e > $OUT/b_${c}_$m.json 2>/dev/null
  tail -1 $OUT/b_${c}_$m.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['phases_ms_per_step']; print('$c $m newton %.4f flux %.3f it %s' % (p['ms_newton'], p['ms_flux_interior'], d.get('newton_iter_max')))"
done; done
