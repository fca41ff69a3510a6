cd $GRAFT_REPO_ROOT
bash tools/gpu_newton_ab.sh nab2 2>&1 | grep -v "lanes4\|warp"
OUT=gpurun_out/s3; mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q --timeout 1500 > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
tail -8 $OUT/pytest_gpu.log
