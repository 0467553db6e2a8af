#!/bin/bash
OUT=gpurun_out/r02d3; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py -q -k "direct or general_radius or wrap" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --engine direct"
for c in heat3d_512 star3d13p_512 star3d19p_512 box3d27p_512; do for s in 0 1; do
  echo "$c star=$s $(CSX_DIRECT3D_STAR=$s timeout 300 $B --config $c 2>/dev/null)" >> $OUT/ab.txt; done; done
