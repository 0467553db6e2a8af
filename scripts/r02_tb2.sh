#!/bin/bash
OUT=gpurun_out/r02t; mkdir -p $OUT
for g in 1 3 4 5 6; do CSX_TB_GEOM=$g timeout 300 python scripts/tb2_parity.py >> $OUT/parity.txt 2>&1; done
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --config heat3d_512"
for g in 1 3 4 5 6 1 3; do echo "geom=$g $(CSX_TB_GEOM=$g timeout 300 $B 2>/dev/null)" >> $OUT/ab.txt; done
