#!/bin/bash
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-sweep3}; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_box.py -q -x > $OUT/pytest_box.log 2>&1; echo "rc=$?" >> $OUT/pytest_box.log; tail -3 $OUT/pytest_box.log
timeout 900 python tools/sweep_box.py C4 "5:80:6:8 5:80:6:8 1:80:6:8 5:100:6:8 11:80:6:8 5:80:5:16 2:80:5:16 1:80:5:16 5:100:5:16 5:80:4:20 5:80:5:12" > $OUT/c4.txt 2>&1
timeout 900 python tools/sweep_box.py C5 "5:80:6:8 1:80:6:8 5:80:5:16 1:80:5:16 11:80:5:16" 3 > $OUT/c5.txt 2>&1
cat $OUT/c4.txt $OUT/c5.txt
