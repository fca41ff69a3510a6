#!/bin/bash
# Round measurement pass: GPU tests, bench lines (C4 default, C5, C4 rate law,
# C3, C3t, reference arm), the ncu launch list and one ncu --set full of the flux kernel.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-round}; mkdir -p $OUT
nvidia-smi -q | grep -i -A3 "clocks$" > $OUT/clocks_before.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -3 $OUT/pytest_gpu.log
timeout 900 python bench.py > $OUT/bench_C4.json 2> $OUT/bench_C4.err; tail -1 $OUT/bench_C4.json | cut -c1-300
timeout 900 python bench.py --config C5 --steps 10 > $OUT/bench_C5.json 2> $OUT/bench_C5.err; tail -1 $OUT/bench_C5.json | cut -c1-300
timeout 900 python bench.py --rate-law --steps 20 --no-cpu-baseline > $OUT/bench_C4_ratelaw.json 2> $OUT/bench_C4_ratelaw.err; tail -1 $OUT/bench_C4_ratelaw.json | cut -c1-300
timeout 900 python bench.py --config C3 --steps 50 > $OUT/bench_C3.json 2> $OUT/bench_C3.err; tail -1 $OUT/bench_C3.json | cut -c1-300
timeout 900 python bench.py --config C3t --steps 20 > $OUT/bench_C3t.json 2> $OUT/bench_C3t.err; tail -1 $OUT/bench_C3t.json | cut -c1-300
timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_reference_C4.json 2> $OUT/bench_reference_C4.err; tail -1 $OUT/bench_reference_C4.json | cut -c1-300
B="python bench.py --no-cpu-baseline --no-e2e"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_C4.csv $B --warmup 3 --steps 2 > $OUT/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux -s 3 -c 1 -o $OUT/prof_flux_C4 $B --steps 1 --warmup 3 > $OUT/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux -s 15 -c 1 -o $OUT/prof_flux_C5 $B --config C5 --steps 1 --warmup 3 > $OUT/ncu_full_C5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux -s 3 -c 1 -o $OUT/prof_flux_C3 $B --config C3 --steps 1 --warmup 3 > $OUT/ncu_full_C3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux -s 3 -c 1 -o $OUT/prof_flux_C3t $B --config C3t --steps 1 --warmup 3 > $OUT/ncu_full_C3t.log 2>&1
echo done
