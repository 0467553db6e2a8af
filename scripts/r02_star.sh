#!/bin/bash
# 3D star shapes: conflict-free DFMA plane loads (CSX_STAR_CF) — parity + A/B bench
OUT=gpurun_out/r02s; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_coverage.py -q -k "3d or star3d" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for c in star3d13p_512 star3d19p_512; do
  for cf in 0 1; do echo "$c cf=$cf $(CSX_STAR_CF=$cf timeout 300 $B --config $c 2>/dev/null)" >> $OUT/ab.txt; done
done
NCU=/usr/local/cuda/bin/ncu
for cf in 0 1; do
CSX_STAR_CF=$cf timeout 600 $NCU --metrics gpu__time_duration.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum --clock-control none -k regex:k_tile3d -s 2 -c 2 --csv python scripts/one_run.py --config star3d13p_512 --T 4 > $OUT/ncu13_cf$cf.csv 2>&1
CSX_STAR_CF=$cf timeout 600 $NCU --metrics gpu__time_duration.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum --clock-control none -k regex:k_tile3d -s 2 -c 2 --csv python scripts/one_run.py --config star3d19p_512 --T 4 > $OUT/ncu19_cf$cf.csv 2>&1
done
