#!/bin/bash
OUT=gpurun_out/r02ch; mkdir -p $OUT
B="python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-comparator"
for c in box2d9p_10240 heat1d_102400000 1d5p_102400000 star2d13p_10240 heat3d_512; do
  echo "$c auto $(timeout 600 $B --config $c 2>/dev/null)" >> $OUT/ab.txt
done
for k in 2 4 6; do echo "box2d9p_10240 k=$k $(CSX_HOST_CHUNKS=$k timeout 600 $B --config box2d9p_10240 2>/dev/null)" >> $OUT/ab.txt; done
for k in 12 16; do echo "heat1d_102400000 k=$k $(CSX_HOST_CHUNKS=$k timeout 600 $B --config heat1d_102400000 2>/dev/null)" >> $OUT/ab.txt; done
