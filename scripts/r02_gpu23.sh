#!/bin/bash
OUT=gpurun_out/r02as; mkdir -p $OUT
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for c in heat1d_10240000 heat1d_102400000; do for tf in 9 11 13 15; do
  echo "$c tf=$tf $(timeout 300 $B --config $c --fuse $tf 2>/dev/null)" >> $OUT/sweep.txt
done; done
for c in 1d5p_10240000 1d5p_102400000; do for tf in 4 5 6 7; do
  echo "$c tf=$tf $(timeout 300 $B --config $c --fuse $tf 2>/dev/null)" >> $OUT/sweep.txt
done; done
