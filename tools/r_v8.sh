cd $GRAFT_REPO_ROOT
OUT=gpurun_out/v8; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > $OUT/pytest_gpu.log 2>&1; tail -2 $OUT/pytest_gpu.log
L=paper_conf_ipps_heislersdms24_b200/libbte.so
bash tools/gpu_libsweep.sh v8 $L "--band-group 4 --dir-chunk 40" "--band-group 5 --dir-chunk 40" "--band-group 6 --dir-chunk 40" "--band-group 7 --dir-chunk 40" "--band-group 8 --dir-chunk 40" "--band-group 6 --dir-chunk 20" "--band-group 6 --dir-chunk 80"
bash tools/gpu_libsweep.sh v8 build_exp/libbte_mb3.so "--band-group 3 --dir-chunk 40" "--band-group 4 --dir-chunk 40" "--band-group 5 --dir-chunk 40" "--band-group 4 --dir-chunk 20" "--band-group 4 --dir-chunk 80"
cat $OUT/sweep.txt
