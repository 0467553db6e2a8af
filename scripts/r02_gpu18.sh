#!/bin/bash
OUT=gpurun_out/r02al; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py -q -k "two_step or (wrap and heat3d)" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log

B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for gg in 1; do for c in heat3d_512 box3d27p_512; do
  echo "geom=$gg $c $(CSX_TB_GEOM=$gg timeout 300 $B --config $c --fuse 2 2>/dev/null)" >> $OUT/sweep.txt
done; done
