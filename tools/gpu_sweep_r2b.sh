#!/bin/bash
# Round-2 sweep b: Newton kernels (C4, C3), box-kernel store variants (cold ncu DRAM bytes), layer range L=16.
cd $GRAFT_REPO_ROOT
OUT=gpurun_out/${1:-sweepb}; mkdir -p $OUT
L=paper_conf_ipps_heislersdms24_b200/libbte.so
for m in thread lanes8 warp; do
  echo "newton $m" >> $OUT/sweep.txt
  BTE_NEWTON=$m bash tools/gpu_libsweep.sh $(basename $OUT) $L "--steps 10" "--config C3 --steps 30"
done
echo "box L=16" >> $OUT/sweep.txt
BTE_BOX_L=16 bash tools/gpu_libsweep.sh $(basename $OUT) $L "--steps 20" "--config C5 --steps 4"
echo "box default" >> $OUT/sweep.txt
bash tools/gpu_libsweep.sh $(basename $OUT) $L "--steps 20" "--config C5 --steps 4"
B="python bench.py --no-cpu-baseline --no-e2e --warmup 3 --steps 1"
for lib in $L exp_libs/libbte_dhint.so exp_libs/libbte_tmastore.so; do
  n=$(basename $lib .so)
  BTE_LIB=$PWD/$lib timeout 600 ncu --set full --clock-control none -k regex:flux -s 3 -c 1 -o $OUT/prof_$n $B > $OUT/ncu_$n.log 2>&1
done
BTE_BOX_L=16 timeout 600 ncu --set full --clock-control none -k regex:flux -s 3 -c 1 -o $OUT/prof_L16 $B > $OUT/ncu_L16.log 2>&1
BTE_BOX_L=16 timeout 900 ncu --set full --clock-control none -k regex:flux -s 15 -c 1 -o $OUT/prof_L16_C5 $B --config C5 > $OUT/ncu_L16_C5.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:flux -s 15 -c 1 -o $OUT/prof_C5 $B --config C5 > $OUT/ncu_C5.log 2>&1
cat $OUT/sweep.txt
