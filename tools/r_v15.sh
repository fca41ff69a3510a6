cd $GRAFT_REPO_ROOT
OUT=gpurun_out/v15; mkdir -p $OUT
L=paper_conf_ipps_heislersdms24_b200/libbte.so
bash tools/gpu_libsweep.sh v15 $L "--band-group 5"
bash tools/gpu_libsweep.sh v15 build_exp/libbte_s6.so "--band-group 5" "--band-group 4"
bash tools/gpu_libsweep.sh v15 build_exp/libbte_s8.so "--band-group 5" "--band-group 4" "--band-group 3" "--band-group 5 --dir-chunk 80"
bash tools/gpu_libsweep.sh v15 build_exp/libbte_s12.so "--band-group 3" "--band-group 4"
cat $OUT/sweep.txt
