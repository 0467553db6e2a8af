#!/bin/bash
OUT=gpurun_out/r02tbh; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_coverage.py -q -k "tb2" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --config heat3d_512"
for rep in 1 2; do for g in t h; do echo "geom=$g $(CSX_TB_GEOM=$g timeout 300 $B 2>/dev/null)" >> $OUT/ab.txt; done; done
