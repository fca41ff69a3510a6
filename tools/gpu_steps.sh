#!/bin/bash
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-steps}; mkdir -p $OUT
(nvidia-smi --query-gpu=timestamp,clocks.sm,clocks.mem,power.draw,clocks_event_reasons.active --format=csv -lms 200 > $OUT/smi.csv 2>&1 &) 
timeout 600 python tools/sweep_box.py C4 "0:0" 10 > $OUT/s10.txt 2>&1
timeout 600 python tools/sweep_box.py C4 "0:0" 50 > $OUT/s50.txt 2>&1
timeout 600 python tools/sweep_box.py C4 "0:0" 200 > $OUT/s200.txt 2>&1
timeout 600 python tools/sweep_box.py C4 "0:0" 10 > $OUT/s10b.txt 2>&1
timeout 900 python tools/shard_flux.py C4 1 2 4 8 > $OUT/shard.txt 2>&1
cat $OUT/s10.txt $OUT/s50.txt $OUT/s200.txt $OUT/s10b.txt $OUT/shard.txt
