cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
B="python bench.py --warmup 3 --no-cpu-baseline --no-e2e"
for bg in 1 2 4 8; do timeout 300 $B --steps 5 --band-group $bg >> gpurun_out/sweep.jsonl 2>>gpurun_out/sweep.err; done
timeout 300 $B --steps 5 --band-group 4 --block-threads 128 >> gpurun_out/sweep.jsonl 2>>gpurun_out/sweep.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv $B --steps 2 > gpurun_out/launches_run.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:flux_kernel -s 6 -c 2 -o gpurun_out/prof_flux $B --steps 1 > gpurun_out/ncu_full.log 2>&1
ls -la gpurun_out
