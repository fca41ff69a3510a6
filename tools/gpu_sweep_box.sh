#!/bin/bash
# Box-kernel work-split sweep: auto planner vs fixed band-rows/directions per CTA,
# then one ncu --set full capture of the box kernel (auto plan).
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-sweep}; mkdir -p $OUT
B="python bench.py --warmup 3 --steps 10 --no-cpu-baseline --no-e2e"
run() { echo -n "$* : " >> $OUT/sweep.txt; timeout 300 $B "$@" 2>>$OUT/sweep.err | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('%.4g upd/s frac %.3f ms %.3f nbb %s chunks %s clk %s %s'%(d['value'],d['roofline']['frac'],d['ms_per_step'],d['band_group'],d['dir_chunks'],d['clocks']['sm_mhz'],d['clocks']['reasons']))" >> $OUT/sweep.txt; }
run
run --band-group 5 --dir-chunk 100
run --band-group 6 --dir-chunk 200
run --band-group 11 --dir-chunk 100
run --band-group 5 --dir-chunk 80
run --band-group 1 --dir-chunk 100
run
run --config C5 --steps 3
timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux -s 0 -c 1 -o $OUT/prof_flux $B --steps 1 --warmup 3 > $OUT/ncu_full.log 2>&1
cat $OUT/sweep.txt
