#!/bin/bash
OUT=gpurun_out/r02am; mkdir -p $OUT
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for v in 1 6 7 8; do for c in box2d25p_10240 star2d9p_10240; do
  echo "v=$v $c $(CSX_TILE_VARIANT=$v timeout 300 $B --config $c 2>/dev/null)" >> $OUT/sweep.txt
done; done
for v in 6 7 8; do CSX_TILE_VARIANT=$v timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "fusion_depths_2d or deep_fusion" > $OUT/t$v.log 2>&1; echo "rc=$?" >> $OUT/t$v.log; done
