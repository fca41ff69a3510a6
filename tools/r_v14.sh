cd $GRAFT_REPO_ROOT
OUT=gpurun_out/v14; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > $OUT/pytest_gpu.log 2>&1; tail -2 $OUT/pytest_gpu.log
L=paper_conf_ipps_heislersdms24_b200/libbte.so
bash tools/gpu_libsweep.sh v14 $L "--band-group 2" "--band-group 5" "--band-group 5 --dir-chunk 20"
bash tools/gpu_libsweep.sh v14 build_exp/libbte_mb1pf.so "--band-group 4" "--band-group 6" "--band-group 8" "--band-group 8 --dir-chunk 20"
bash tools/gpu_libsweep.sh v14 build_exp/libbte_nopf.so "--band-group 5" "--band-group 5 --dir-chunk 20"
cat $OUT/sweep.txt
