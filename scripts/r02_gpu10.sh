#!/bin/bash
OUT=gpurun_out/r02j; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "s2r" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --engine tc_s2r"
for ws in 1 0; do
for c in box2d9p_10240 box2d49p_10240 box2d25p_10240; do
  echo "ws=$ws $c $(CSX_S2R_WS=$ws timeout 600 $B --config $c 2>/dev/null)" >> $OUT/s2r.txt
done; done
python scripts/dmma_counters.py --out $OUT/dmma.json box2d9p_10240:tc_s2r box2d49p_10240:tc_s2r box2d9p_10240:direct heat2d_10240:direct box2d49p_10240:direct > $OUT/dmma.log 2>&1
