#!/bin/bash
# Round-2 sweeps: generic-kernel ring depth / work split on C3t, Newton lanes per cell on C4 / C3.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-sweep}; mkdir -p $OUT
for lib in exp_libs/libbte_g3.so exp_libs/libbte_g4.so exp_libs/libbte_g6.so; do
  bash tools/gpu_libsweep.sh $(basename $OUT) $lib "--config C3t --steps 20" "--config C3t --steps 20 --dir-chunk 80" "--config C3t --steps 20 --band-group 2" "--config C3t --steps 20 --dir-chunk 100 --band-group 2"
done
for m in thread lanes4 lanes8 lanes16 warp; do
  echo "newton $m" >> $OUT/sweep.txt
  BTE_NEWTON=$m bash tools/gpu_libsweep.sh $(basename $OUT) paper_conf_ipps_heislersdms24_b200/libbte.so "--steps 10" "--config C3 --steps 30"
done
cat $OUT/sweep.txt
