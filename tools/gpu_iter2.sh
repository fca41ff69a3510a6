#!/bin/bash
# tests + bench sweep + one ncu capture. usage: bash tools/gpu_iter2.sh TAG "NCU-ARGS" "ARGS1" "ARGS2" ...
cd $GRAFT_REPO_ROOT
TAG=$1; NCUA=$2; shift 2
OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > $OUT/pytest_gpu.log 2>&1
tail -3 $OUT/pytest_gpu.log
bash tools/gpu_sweep.sh $TAG "$@" > /dev/null
cat $OUT/sweep.txt | grep -v "^=="
if [ -n "$NCUA" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux -s 0 -c 1 -o $OUT/prof \
   python bench.py --warmup 3 --steps 1 --no-cpu-baseline --no-e2e $NCUA > $OUT/ncu.log 2>&1
fi
