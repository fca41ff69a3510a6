cd $GRAFT_REPO_ROOT
OUT=gpurun_out/v11; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > $OUT/pytest_gpu.log 2>&1; tail -2 $OUT/pytest_gpu.log
L=paper_conf_ipps_heislersdms24_b200/libbte.so
bash tools/gpu_libsweep.sh v11 $L "--band-group 8" "--band-group 4" "--band-group 8 --dir-chunk 20" "--band-group 6"
bash tools/gpu_libsweep.sh v11 build_exp/libbte_mb3.so "--band-group 4" "--band-group 4 --no-tma" "--band-group 4 --dir-chunk 20"
cat $OUT/sweep.txt
timeout 900 ncu --set full --clock-control none -k regex:flux -s 0 -c 1 -o $OUT/prof python bench.py --warmup 3 --steps 1 --no-cpu-baseline --no-e2e --band-group 8 > $OUT/ncu.log 2>&1
