#!/bin/bash
OUT=gpurun_out/r02t3; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_coverage.py -q -k "tb2" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --config heat3d_512"
for rep in 1 2; do for g in t a b c; do echo "geom=$g $(CSX_TB_GEOM=$g timeout 300 $B 2>/dev/null)" >> $OUT/ab.txt; done; done
for g in t a; do echo "box geom=$g $(CSX_TB_GEOM=$g timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --config box3d27p_512 --fuse 2 2>/dev/null)" >> $OUT/ab.txt; done
