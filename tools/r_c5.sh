cd $GRAFT_REPO_ROOT
OUT=gpurun_out/c5; mkdir -p $OUT
nvidia-smi --query-gpu=memory.total,memory.free --format=csv > $OUT/mem.txt
timeout 1500 python bench.py --config C5 --steps 10 --warmup 3 --no-e2e --ic-eps 0.0 > $OUT/bench_c5.json 2> $OUT/bench_c5.err
cat $OUT/bench_c5.json; tail -5 $OUT/bench_c5.err
timeout 900 python bench.py --config C3 --steps 50 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/bench_c3.json 2> $OUT/bench_c3.err
cat $OUT/bench_c3.json; tail -3 $OUT/bench_c3.err
