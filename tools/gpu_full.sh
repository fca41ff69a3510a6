#!/bin/bash
# Full GPU pass: sanitizers on the box kernel, the whole GPU suite, bench C4 + C5,
# the ncu launch list and one ncu --set full capture of the dominant kernel.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-full}; mkdir -p $OUT
K="test_box_fig1_ragged or test_box_all_specular or test_box_slab_rotation"
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python -m pytest tests/test_gpu_box.py -q -x -k "$K" > $OUT/san_$tool.log 2>&1
  echo "$tool rc=$?" >> $OUT/san_$tool.log; tail -3 $OUT/san_$tool.log
done
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 900 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -15 $OUT/pytest_gpu.log
B="python bench.py --no-cpu-baseline --no-e2e"
timeout 600 python bench.py > $OUT/bench_C4.json 2> $OUT/bench_C4.err; tail -1 $OUT/bench_C4.json
timeout 900 $B --config C5 --steps 5 --warmup 3 > $OUT/bench_C5.json 2> $OUT/bench_C5.err; tail -1 $OUT/bench_C5.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_C4.csv $B --warmup 3 --steps 2 > $OUT/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux -s 0 -c 1 -o $OUT/prof_flux $B --steps 1 --warmup 1 > $OUT/ncu_full.log 2>&1
echo done
