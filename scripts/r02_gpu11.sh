#!/bin/bash
OUT=gpurun_out/r02k; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "s2r" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --engine tc_s2r"
for c in box2d9p_10240 box2d49p_10240 box2d25p_10240 heat2d_10240; do
  echo "ws=1 $c $(timeout 600 $B --config $c 2>/dev/null)" >> $OUT/s2r.txt
done
python scripts/dmma_counters.py --out $OUT/dmma.json box2d9p_10240:tc_s2r box2d25p_10240:tc_s2r > $OUT/dmma.log 2>&1
