#!/bin/bash
OUT=gpurun_out/r02q; mkdir -p $OUT
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for v in 9 a b; do for c in heat3d_512 box3d27p_512; do
  echo "v=$v $c $(CSX_TILE3D_VARIANT=$v timeout 300 $B --config $c 2>/dev/null)" >> $OUT/sweep.txt
  CSX_TILE3D_VARIANT=$v /usr/local/cuda/bin/ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:k_tile3d -s 2 -c 1 python scripts/one_run.py --config $c --T 6 > $OUT/ncu_${c}_v$v.txt 2>&1
done; done
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "tile_variants" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
bash scripts/r02_sanitize.sh
