#!/bin/bash
# ncu --set full of the first main flux launch for each bench arg set.
# usage: bash tools/gpu_ncu.sh TAG "ARGS1" "ARGS2" ...
cd $GRAFT_REPO_ROOT
TAG=$1; shift
OUT=gpurun_out/$TAG; mkdir -p $OUT
i=0
for a in "$@"; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux -s 0 -c 1 -o $OUT/prof_$i \
      python bench.py --warmup 3 --steps 1 --no-cpu-baseline --no-e2e $a > $OUT/ncu_$i.log 2>&1
  echo "$i: $a" >> $OUT/index.txt
  i=$((i+1))
done
cat $OUT/index.txt
