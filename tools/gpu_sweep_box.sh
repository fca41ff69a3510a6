#!/bin/bash
# Box-kernel work-split sweep on C4 (and C5): band-rows per CTA x directions per CTA.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-sweep}; mkdir -p $OUT
CFG=${2:-C4}
B="python bench.py --config $CFG --warmup 3 --steps 5 --no-cpu-baseline --no-e2e"
for nbb in ${3:-5 11 1}; do for dc in ${4:-100 80 200 40}; do
  echo -n "nbb=$nbb dc=$dc " >> $OUT/sweep.txt
  timeout 300 $B --band-group $nbb --dir-chunk $dc 2>>$OUT/sweep.err | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('%.4g upd/s frac %.3f ms %.3f'%(d['value'],d['roofline']['frac'],d['ms_per_step']))" >> $OUT/sweep.txt
done; done
cat $OUT/sweep.txt
