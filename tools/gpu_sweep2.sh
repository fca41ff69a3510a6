#!/bin/bash
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-sweep2}; mkdir -p $OUT
timeout 900 python tools/sweep_box.py C4 "5:80 5:80 5:60 5:40 5:120 4:80 3:80 2:80 1:80 1:40 6:80 7:80 5:20 0:0" > $OUT/c4.txt 2>&1
timeout 900 python tools/sweep_box.py C5 "5:80 1:80 3:80 0:0" 3 > $OUT/c5.txt 2>&1
cat $OUT/c4.txt $OUT/c5.txt
