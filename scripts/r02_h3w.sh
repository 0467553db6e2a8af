#!/bin/bash
OUT=gpurun_out/r02h3w; mkdir -p $OUT
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --config heat3d_512 --fuse 1"
for v in 9 z u; do echo "heat3d_tf1 v=$v $(CSX_TILE3D_VARIANT=$v timeout 300 $B 2>/dev/null)" >> $OUT/ab.txt; done
for v in 0 z u; do echo "box3d27p v=$v $(CSX_TILE3D_VARIANT=$v timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --config box3d27p_512 2>/dev/null)" >> $OUT/ab.txt; done
NCU=/usr/local/cuda/bin/ncu
for v in 9 z u; do CSX_TILE3D_VARIANT=$v timeout 600 $NCU --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:k_tile3d -s 2 -c 1 --csv python scripts/one_run.py --config heat3d_512 --T 6 --fuse 1 > $OUT/ncu_$v.csv 2>&1; done
