#!/bin/bash
OUT=gpurun_out/r02i; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "direct_comparator or tile_variants" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e"
for c in box2d9p_10240 heat2d_10240 star2d9p_10240 box2d25p_10240 star2d13p_10240 box2d49p_10240 star2d13p_10240_tf2; do
  timeout 600 $B --config $c >> $OUT/bench2d.jsonl 2>> $OUT/bench.err
done
for v in 5 7; do
  echo "v=$v $(CSX_TILE3D_VARIANT=$v timeout 300 $B --no-comparator --config heat3d_512 2>/dev/null)" >> $OUT/heat3d_sweep.txt
  CSX_TILE3D_VARIANT=$v /usr/local/cuda/bin/ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --clock-control none -k regex:k_tile3d -s 2 -c 1 python scripts/one_run.py --config heat3d_512 --T 12 > $OUT/ncu_heat3d_v$v.txt 2>&1
done
