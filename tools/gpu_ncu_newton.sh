#!/bin/bash
# ncu --set full of the temperature-solve kernels (C4: thread per cell, C3: lanes + finish).
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-nw}; mkdir -p $OUT
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "nccl or one_rank" > $OUT/pytest.log 2>&1; tail -2 $OUT/pytest.log
B="python bench.py --no-cpu-baseline --no-e2e --warmup 3 --steps 1"
for c in C4 C3; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"newton|sum_slots" -s 6 -c 3 -o $OUT/prof_$c $B --config $c > $OUT/ncu_$c.log 2>&1
  ncu -i $OUT/prof_$c.ncu-rep --page raw --csv > $OUT/raw_$c.csv 2>/dev/null
  ncu -i $OUT/prof_$c.ncu-rep --page source --csv --print-source sass > $OUT/src_$c.csv 2>/dev/null; gzip -f $OUT/src_$c.csv
  python tools/ncu_summary.py full $OUT/raw_$c.csv $OUT/sum_$c.json --config $c
done
for spec in "C4 20" "C3 50"; do
  set -- $spec
  timeout 600 python bench.py --config $1 --steps $2 --no-cpu-baseline --no-e2e > $OUT/bench_$1.json 2> $OUT/bench_$1.err
  tail -1 $OUT/bench_$1.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', d['value'], d['phases_ms_per_step'], d.get('newton_iter_max'))"
done
