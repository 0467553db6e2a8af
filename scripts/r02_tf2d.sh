#!/bin/bash
OUT=gpurun_out/r02tf; mkdir -p $OUT
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -k "run_host" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for rep in 1 2; do for tf in 3 2 4; do
  echo "box2d9p tf=$tf $(timeout 300 $B --config box2d9p_10240 --fuse $tf 2>/dev/null)" >> $OUT/ab.txt
  echo "heat2d tf=$tf $(timeout 300 $B --config heat2d_10240 --fuse $tf 2>/dev/null)" >> $OUT/ab.txt
done; done
