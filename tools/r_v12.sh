cd $GRAFT_REPO_ROOT
OUT=gpurun_out/v12; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 > $OUT/pytest_gpu.log 2>&1; tail -2 $OUT/pytest_gpu.log
python tools/copy_calib.py > $OUT/copy.txt 2>&1; cat $OUT/copy.txt
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -s 3 -c 1 python tools/copy_calib.py > $OUT/copy_ncu.txt 2>&1
grep -E "dram__|gpu__time" $OUT/copy_ncu.txt
L=paper_conf_ipps_heislersdms24_b200/libbte.so
bash tools/gpu_libsweep.sh v12 $L "--band-group 4" "--band-group 5" "--band-group 4 --dir-chunk 20" "--band-group 3 --dir-chunk 20" "--band-group 8 --no-tma --dir-chunk 20"
cat $OUT/sweep.txt
timeout 900 ncu --set full --clock-control none -k regex:flux -s 0 -c 1 -o $OUT/prof python bench.py --warmup 3 --steps 1 --no-cpu-baseline --no-e2e --band-group 4 --dir-chunk 20 > $OUT/ncu.log 2>&1
