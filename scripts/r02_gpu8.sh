#!/bin/bash
OUT=gpurun_out/r02h; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "direct_comparator" > $OUT/d2.log 2>&1; echo "rc=$?" >> $OUT/d2.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for c in box2d25p_10240 box2d49p_10240 star2d13p_10240; do
  for tf in 1 2; do
    for env in "CSX_DIRECT2D=wf" "CSX_DIRECT2D=smem"; do
      echo "$c $env tf=$tf $(env $env timeout 300 $B --config $c --engine direct --fuse $tf 2>/dev/null)" >> $OUT/d2_sweep.txt
    done
  done
done
