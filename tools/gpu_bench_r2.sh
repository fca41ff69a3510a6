#!/bin/bash
# Bench lines of every workload (+ reference arm, board power) into gpurun_out/TAG.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-r02b}; mkdir -p $OUT
timeout 900 python bench.py > $OUT/bench_C4.json 2> $OUT/bench_C4.err; tail -1 $OUT/bench_C4.json | cut -c1-200
timeout 900 python bench.py --config C5 --steps 10 > $OUT/bench_C5.json 2> $OUT/bench_C5.err; tail -1 $OUT/bench_C5.json | cut -c1-200
timeout 900 python bench.py --rate-law --steps 20 --no-cpu-baseline > $OUT/bench_C4_ratelaw.json 2> $OUT/bench_C4_ratelaw.err
timeout 900 python bench.py --config C3 --steps 50 > $OUT/bench_C3.json 2> $OUT/bench_C3.err
timeout 900 python bench.py --config C3t --steps 20 > $OUT/bench_C3t.json 2> $OUT/bench_C3t.err
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $OUT/bench_reference_C4.json 2> $OUT/bench_reference_C4.err
timeout 300 python tools/power_probe.py > $OUT/power_C4.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
B="python bench.py --no-cpu-baseline --no-e2e --warmup 3"
timeout 1200 ncu --set full --clock-control none -k regex:flux -s 18 -c 1 -o $OUT/prof_C5 $B --steps 1 --config C5 > $OUT/ncu_C5.log 2>&1
ncu -i $OUT/prof_C5.ncu-rep --page raw --csv > $OUT/raw_C5.csv 2>/dev/null; rm -f $OUT/prof_C5.ncu-rep
