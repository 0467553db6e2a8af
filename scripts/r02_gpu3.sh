#!/bin/bash
# round 2, call 3: 2D register-wavefront comparator (parity, variants, sweep), 3D star rings
OUT=gpurun_out/r02c; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "direct_comparator_2d" > $OUT/d2.log 2>&1; echo "rc=$?" >> $OUT/d2.log
timeout 600 python -m pytest tests/test_gpu_coverage.py -q -k "general_radius or (wrap and (3d or direct))" > $OUT/r3d.log 2>&1; echo "rc=$?" >> $OUT/r3d.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator"
for tf in 1 2 3 4; do
  for env in "CSX_DIRECT2D_V=2" "CSX_DIRECT2D_V=4" "CSX_DIRECT2D_MINB=2" "CSX_DIRECT2D=smem"; do
    echo "$env tf=$tf $(env $env timeout 300 $B --config box2d9p_10240 --engine direct --fuse $tf 2>/dev/null)" >> $OUT/d2_sweep.txt
  done
done
for c in star3d13p_512 star3d19p_512 box3d125p_512 box3d343p_512; do
  timeout 300 $B --config $c >> $OUT/bench3d.jsonl 2>> $OUT/bench.err
done
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline >> $OUT/bench_c2.jsonl 2>> $OUT/bench.err
