#!/bin/bash
OUT=gpurun_out/r02ao; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py -q -k "s2r or 3d" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --engine tc_s2r"
for ws in 1 0; do for c in box3d27p_512 heat3d_512; do
  echo "ws=$ws $c $(CSX_S2R_WS=$ws timeout 300 $B --config $c 2>/dev/null)" >> $OUT/sweep.txt
done; done
