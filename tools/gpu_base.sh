#!/bin/bash
# Baseline GPU pass: parity tests, the default bench line, and the ncu launch list.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-base}; mkdir -p $OUT
nvidia-smi -L > $OUT/gpu.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x --timeout 900 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -3 $OUT/pytest_gpu.log
timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err; tail -1 $OUT/bench.json
