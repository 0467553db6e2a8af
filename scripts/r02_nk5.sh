#!/bin/bash
OUT=gpurun_out/r02nk5; mkdir -p $OUT
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --config box2d9p_10240"
for v in 1 6 7 8 2 0 1; do echo "v=$v $(CSX_TILE_VARIANT=$v timeout 300 $B 2>/dev/null)" >> $OUT/ab.txt; done
