#!/bin/bash
# C5 box-kernel orbit-chunk sweep: flux time (sweep_box, equilibrium IC) and DRAM bytes of one launch (ncu).
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-c5oc}; mkdir -p $OUT
for oc in 20 10 5 25; do
  BTE_BOX_OC=$oc timeout 600 python tools/sweep_box.py C5 "0:0:5:8" 5 2>&1 | grep -v Warn | sed "s/^/oc $oc: /"
  BTE_BOX_OC=$oc timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:flux -s 7 -c 1 --csv python bench.py --config C5 --warmup 1 --steps 1 --no-cpu-baseline --no-e2e 2>/dev/null | grep -E "dram__bytes|gpu__time" | awk -F'","' '{print "oc '$oc'", $(NF-2), $(NF-1), $NF}'
done
