#!/bin/bash
OUT=gpurun_out/r02g; mkdir -p $OUT
timeout 300 python scripts/dbg_wf.py > $OUT/dbg_wf.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "direct_comparator_2d" > $OUT/d2.log 2>&1; echo "rc=$?" >> $OUT/d2.log
timeout 900 python -m pytest tests/test_gpu_coverage.py -q -k "wrap and direct" > $OUT/wrap.log 2>&1; echo "rc=$?" >> $OUT/wrap.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for tf in 1 2 3 4; do
  for env in "CSX_DIRECT2D_UNR=0" "CSX_DIRECT2D_UNR=1" "CSX_DIRECT2D_V=4"; do
    echo "$env tf=$tf $(env $env timeout 300 $B --config box2d9p_10240 --engine direct --fuse $tf 2>/dev/null)" >> $OUT/d2_sweep.txt
  done
done
for c in box2d25p_10240 star2d9p_10240; do echo "$c $(timeout 300 $B --config $c --engine direct 2>/dev/null)" >> $OUT/d2_sweep.txt; done
