#!/bin/bash
OUT=gpurun_out/r02w; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_coverage.py -q -k "tb2 or 3d" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for c in heat1d_102400000 1d5p_102400000 heat1d_10240000; do
  for v in 0 1 2 3 4 5 6 7; do echo "$c v=$v $(CSX_TILE1D_VARIANT=$v timeout 300 $B --config $c 2>/dev/null)" >> $OUT/sweep.txt; done
done
for g in 7 8 1; do echo "heat3d g=$g $(CSX_TB_GEOM=$g timeout 300 $B --config heat3d_512 2>/dev/null)" >> $OUT/sweep.txt; done
