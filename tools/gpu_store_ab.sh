#!/bin/bash
# Box-kernel store variants: sustained bench (C4 x2, C5) + cold ncu DRAM bytes (raw CSV) per library.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-store}; shift; mkdir -p $OUT
B="python bench.py --no-cpu-baseline --no-e2e --warmup 3"
for lib in "$@"; do
  n=$(basename $lib .so)
  for rep in 1 2; do
    BTE_LIB=$PWD/$lib timeout 300 $B --steps 20 > $OUT/${n}_C4_$rep.json 2>/dev/null
  done
  BTE_LIB=$PWD/$lib timeout 600 $B --steps 4 --config C5 > $OUT/${n}_C5.json 2>/dev/null
  BTE_LIB=$PWD/$lib timeout 600 ncu --set full --clock-control none -k regex:flux -s 3 -c 1 -o $OUT/p_$n $B --steps 1 > /dev/null 2>&1
  ncu -i $OUT/p_$n.ncu-rep --page raw --csv > $OUT/raw_${n}_C4.csv 2>/dev/null; rm -f $OUT/p_$n.ncu-rep
  python - $n $OUT <<'PY'
import json,sys,glob
n,o=sys.argv[1],sys.argv[2]
for f in sorted(glob.glob(f"{o}/{n}_C*.json")):
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1]); p=d['phases_ms_per_step']
        print(f.split('/')[-1], '%.4g upd/s'%d['value'], 'flux %.3f'%p['ms_flux_interior'], 'frac %.3f'%d['roofline']['frac'], d['clocks'].get('sm_mhz'), d['clocks'].get('reasons'))
    except Exception as e: print(f, 'FAILED', e)
PY
done
