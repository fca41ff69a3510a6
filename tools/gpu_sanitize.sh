cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-san}; mkdir -p $OUT
for t in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $t --error-exitcode 9 python tools/sanitize_run.py > $OUT/$t.log 2>&1
  echo "$t exit $?"; tail -4 $OUT/$t.log
done
