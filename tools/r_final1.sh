cd $GRAFT_REPO_ROOT
OUT=gpurun_out/f1; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q --timeout 600 > $OUT/pytest_gpu.log 2>&1; tail -2 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; cat $OUT/bench.json
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_ref.json 2> $OUT/bench_ref.err; cat $OUT/bench_ref.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv python bench.py --warmup 3 --steps 2 --no-cpu-baseline --no-e2e > $OUT/launches_run.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux -s 0 -c 1 -o $OUT/prof_flux python bench.py --warmup 3 --steps 1 --no-cpu-baseline --no-e2e > $OUT/ncu_full.log 2>&1
ls $OUT
