#!/bin/bash
OUT=gpurun_out/r02last; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "tile_variants" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for c in heat1d_102400000 heat1d_10240000 1d5p_102400000; do for h in 1 0; do
  echo "$c hint=$h $(CSX_TMA_HINT=$h timeout 300 $B --config $c 2>/dev/null)" >> $OUT/ab.txt; done; done
