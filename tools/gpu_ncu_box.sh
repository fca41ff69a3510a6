#!/bin/bash
# ncu --set full of the box kernel for a few launch configurations (band_group:dir_chunk:stages:L)
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-ncubox}; mkdir -p $OUT
shift
for c in "$@"; do
  n=$(echo $c | tr ':' '_')
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux_box -s 3 -c 1 -o $OUT/box_$n \
     python tools/sweep_box.py C4 "$c" 1 > $OUT/ncu_$n.log 2>&1
done
ls $OUT
