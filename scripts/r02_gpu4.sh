#!/bin/bash
OUT=gpurun_out/r02d; mkdir -p $OUT
timeout 300 python scripts/dbg_wf.py > $OUT/dbg_wf.txt 2>&1
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --config heat3d_512"
for env in "CSX_TILE3D_VARIANT=9" "CSX_TILE3D_VARIANT=4" "CSX_TILE3D_VARIANT=6" "CSX_TMA_HINT=0" "CSX_TMA_HINT=1" "CSX_TMA_PROMO=256" "CSX_TMA_PROMO=128" "CSX_TILE3D_VARIANT=4 CSX_TMA_HINT=0" "CSX_TILE3D_VARIANT=4 CSX_TMA_PROMO=256"; do
  echo "$env $(env $env timeout 300 $B 2>/dev/null)" >> $OUT/heat3d_sweep.txt
done
for v in 4 6; do
 CSX_TILE3D_VARIANT=$v timeout 300 python scripts/one_run.py --config heat3d_512 --T 3 > /dev/null 2>&1
 CSX_TILE3D_VARIANT=$v /usr/local/cuda/bin/ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:k_tile3d -s 2 -c 1 python scripts/one_run.py --config heat3d_512 --T 12 > $OUT/ncu_heat3d_v$v.txt 2>&1
done
/usr/local/cuda/bin/ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:k_tile3d -s 2 -c 1 python scripts/one_run.py --config heat3d_512 --T 12 > $OUT/ncu_heat3d_def.txt 2>&1
