#!/bin/bash
OUT=gpurun_out/r02w; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py -q -k "two_step or (wrap and heat3d) or general_radius_variants" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for tb in 0; do for c in heat3d_512 box3d27p_512; do
  echo "tb=$tb $c $(CSX_TB=$tb timeout 300 $B --config $c --fuse 2 2>/dev/null)" >> $OUT/sweep.txt
done; done
/usr/local/cuda/bin/ncu --set full --clock-control none -k regex:k_tile3d_tb2 -s 2 -c 1 -o $OUT/prof_tb2 -f python scripts/one_run.py --config heat3d_512 --T 12 --fuse 2 > /dev/null 2>&1; python scripts/ncu_brief.py $OUT/prof_tb2.ncu-rep > $OUT/brief_tb2.txt 2>&1; rm -f $OUT/prof_tb2.ncu-rep
