cd $GRAFT_REPO_ROOT
OUT=gpurun_out/s1; mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q --timeout 1500 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -3 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -1 $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench_C4.json 2> $OUT/bench_C4.err; tail -1 $OUT/bench_C4.json | cut -c1-600
timeout 900 python bench.py --config C3t --steps 20 --no-cpu-baseline > $OUT/bench_C3t.json 2> $OUT/bench_C3t.err; tail -1 $OUT/bench_C3t.json | cut -c1-300
timeout 900 python bench.py --config C5 --steps 10 --no-cpu-baseline > $OUT/bench_C5.json 2> $OUT/bench_C5.err; tail -1 $OUT/bench_C5.json | cut -c1-300
