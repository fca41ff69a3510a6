cd $GRAFT_REPO_ROOT
OUT=gpurun_out/v13; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > $OUT/pytest_gpu.log 2>&1; tail -2 $OUT/pytest_gpu.log
L=paper_conf_ipps_heislersdms24_b200/libbte.so
bash tools/gpu_libsweep.sh v13 $L "" "--band-group 4" "--band-group 6" "--band-group 5 --dir-chunk 20" "--band-group 5 --dir-chunk 80" "--config C5 --ic-eps 0 --steps 5"
cat $OUT/sweep.txt
timeout 900 ncu --set full --clock-control none -k regex:flux -s 0 -c 1 -o $OUT/prof python bench.py --warmup 3 --steps 1 --no-cpu-baseline --no-e2e > $OUT/ncu.log 2>&1
