#!/bin/bash
OUT=gpurun_out/r02n; mkdir -p $OUT
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for ko in 1; do for c in star3d13p_512 box3d125p_512 star3d19p_512 box3d343p_512; do
  echo "ko=$ko $c $(CSX_TILE3D_KO=$ko timeout 600 $B --config $c 2>/dev/null)" >> $OUT/ko.txt
done; done
CSX_TILE3D_KO=1 timeout 900 python -m pytest tests/test_gpu_coverage.py -q -k "general_radius or (wrap and 3d)" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
