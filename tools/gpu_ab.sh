#!/bin/bash
# A/B of two library builds on the same box, interleaved: sweep_box.py combos per lib.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-ab}; mkdir -p $OUT
A=$2; B=$3; CFG=$4; COMBOS=$5; STEPS=${6:-10}
for r in 1 2; do
  echo "== A $A" >> $OUT/ab.txt; BTE_LIB=$PWD/$A timeout 600 python tools/sweep_box.py $CFG "$COMBOS" $STEPS >> $OUT/ab.txt 2>&1
  echo "== B $B" >> $OUT/ab.txt; BTE_LIB=$PWD/$B timeout 600 python tools/sweep_box.py $CFG "$COMBOS" $STEPS >> $OUT/ab.txt 2>&1
done
cat $OUT/ab.txt
