#!/bin/bash
OUT=gpurun_out/r02r; mkdir -p $OUT
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for v in 9 8 0; do echo "v=$v heat3d $(CSX_TILE3D_VARIANT=$v timeout 300 $B --config heat3d_512 2>/dev/null)" >> $OUT/sweep.txt; done
for c in star3d13p_512 star3d19p_512 box3d27p_512; do echo "$c $(timeout 300 $B --config $c 2>/dev/null)" >> $OUT/sweep.txt; done
echo "g8 star3d13p $(CSX_TILE3D5_G8=1 timeout 300 $B --config star3d13p_512 2>/dev/null)" >> $OUT/sweep.txt
echo "g8 box3d125p $(CSX_TILE3D5_G8=1 timeout 300 $B --config box3d125p_512 2>/dev/null)" >> $OUT/sweep.txt
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py -q -k "3d" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
