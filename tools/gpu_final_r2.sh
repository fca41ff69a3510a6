#!/bin/bash
# Round-2 measurement pass (one B200): GPU suite, smoke, bench lines per workload,
# the reference arm, ncu launch list and --set full of the flux kernel per config
# (exported to CSV on the box), compute-sanitizer, board power.
# usage: bash tools/gpu_final_r2.sh TAG [quick]
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-r02}; mkdir -p $OUT
MODE=$2  # (the loops below reuse the positional parameters)
nvidia-smi -q | grep -i -A3 "clocks$" > $OUT/clocks_before.txt 2>&1
timeout 2400 python -m pytest tests -m gpu -q --timeout 1500 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -3 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench_C4.json 2> $OUT/bench_C4.err; tail -1 $OUT/bench_C4.json | cut -c1-400
timeout 900 python bench.py --config C5 --steps 10 > $OUT/bench_C5.json 2> $OUT/bench_C5.err; tail -1 $OUT/bench_C5.json | cut -c1-300
timeout 900 python bench.py --rate-law --steps 20 --no-cpu-baseline > $OUT/bench_C4_ratelaw.json 2> $OUT/bench_C4_ratelaw.err; tail -1 $OUT/bench_C4_ratelaw.json | cut -c1-300
timeout 900 python bench.py --config C3 --steps 50 > $OUT/bench_C3.json 2> $OUT/bench_C3.err; tail -1 $OUT/bench_C3.json | cut -c1-300
timeout 900 python bench.py --config C3t --steps 20 > $OUT/bench_C3t.json 2> $OUT/bench_C3t.err; tail -1 $OUT/bench_C3t.json | cut -c1-300
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $OUT/bench_reference_C4.json 2> $OUT/bench_reference_C4.err; tail -1 $OUT/bench_reference_C4.json | cut -c1-300
timeout 300 python tools/power_probe.py > $OUT/power_C4.txt 2>&1
B="python bench.py --no-cpu-baseline --no-e2e --warmup 3"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_C4.csv $B --steps 2 > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_C3.csv $B --steps 2 --config C3 > /dev/null 2>&1
for spec in "C4 3" "C5 15" "C3 3" "C3t 3"; do
  set -- $spec
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:flux -s $2 -c 1 -o $OUT/prof_$1 $B --steps 1 --config $1 > $OUT/ncu_$1.log 2>&1
  ncu -i $OUT/prof_$1.ncu-rep --page raw --csv > $OUT/raw_$1.csv 2>/dev/null
  ncu -i $OUT/prof_$1.ncu-rep --page source --csv --print-source sass > $OUT/src_$1.csv 2>/dev/null; gzip -f $OUT/src_$1.csv
  [ "$1" = "C4" ] || rm -f $OUT/prof_$1.ncu-rep
done
for c in C4 C3; do  # the temperature-solve kernels
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"newton|sum_slots" -s 3 -c 1 -o $OUT/newton_$c $B --steps 1 --config $c > $OUT/ncu_newton_$c.log 2>&1
  ncu -i $OUT/newton_$c.ncu-rep --page raw --csv > $OUT/raw_newton_$c.csv 2>/dev/null; rm -f $OUT/newton_$c.ncu-rep
done
if [ "$MODE" != "quick" ]; then bash tools/gpu_sanitize.sh $(basename $OUT)/san; fi
du -sh $OUT
echo done
