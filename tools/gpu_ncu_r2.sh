#!/bin/bash
# ncu evidence (round 2): launch lists (C4, C3) and --set full of the flux kernel per config,
# exported to CSV on the box (raw + source pages) so the merged gpurun_out stays small.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-ncu}; mkdir -p $OUT
B="python bench.py --no-cpu-baseline --no-e2e --warmup 3"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_C4.csv $B --steps 2 > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_C3.csv $B --steps 2 --config C3 > /dev/null 2>&1
for spec in "C4 3" "C5 15" "C3 3" "C3t 3"; do
  set -- $spec
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:flux -s $2 -c 1 -o $OUT/prof_$1 $B --steps 1 --config $1 > $OUT/ncu_$1.log 2>&1
  ncu -i $OUT/prof_$1.ncu-rep --page raw --csv > $OUT/raw_$1.csv 2>/dev/null
  ncu -i $OUT/prof_$1.ncu-rep --page source --csv --print-source sass > $OUT/src_$1.csv 2>/dev/null
  gzip -f $OUT/src_$1.csv
  [ "$1" = "C4" ] || rm -f $OUT/prof_$1.ncu-rep
done
ls -la $OUT
