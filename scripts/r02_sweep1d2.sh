#!/bin/bash
OUT=gpurun_out/r02w2; mkdir -p $OUT
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for tf in 7 9 11 12 13 14 15; do for v in 0 3 6; do
  echo "heat1d_102400000 tf=$tf v=$v $(CSX_TILE1D_VARIANT=$v timeout 300 $B --config heat1d_102400000 --fuse $tf 2>/dev/null)" >> $OUT/sweep.txt; done; done
for tf in 4 5 6 7; do for v in 0 3 6; do
  echo "1d5p_102400000 tf=$tf v=$v $(CSX_TILE1D_VARIANT=$v timeout 300 $B --config 1d5p_102400000 --fuse $tf 2>/dev/null)" >> $OUT/sweep.txt; done; done
for tf in 11 13 15; do for v in 0 6; do
  echo "heat1d_10240000 tf=$tf v=$v $(CSX_TILE1D_VARIANT=$v timeout 300 $B --config heat1d_10240000 --fuse $tf 2>/dev/null)" >> $OUT/sweep.txt; done; done
for tf in 5 7; do for v in 0 6; do
  echo "1d5p_10240000 tf=$tf v=$v $(CSX_TILE1D_VARIANT=$v timeout 300 $B --config 1d5p_10240000 --fuse $tf 2>/dev/null)" >> $OUT/sweep.txt; done; done
