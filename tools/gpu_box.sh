#!/bin/bash
# Box-kernel iteration: its parity tests first (stop on failure), then the bench line.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-box}; mkdir -p $OUT
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_gpu_box.py -q -x -k "fig1_ragged and 34" > $OUT/sanitize.log 2>&1; echo "sanitize rc=$?" >> $OUT/sanitize.log
tail -5 $OUT/sanitize.log
timeout 900 python -m pytest tests/test_gpu_box.py -q -x --timeout 300 > $OUT/pytest_box.log 2>&1; echo "rc=$?" >> $OUT/pytest_box.log
tail -15 $OUT/pytest_box.log
timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e > $OUT/bench.json 2> $OUT/bench.err; tail -1 $OUT/bench.json; tail -3 $OUT/bench.err
