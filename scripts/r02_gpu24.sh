#!/bin/bash
OUT=gpurun_out/r02au; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py -q -k "s2r" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --engine tc_s2r"
for c in box2d9p_10240 box2d49p_10240; do echo "$c $(timeout 300 $B --config $c 2>/dev/null)" >> $OUT/sweep.txt; done
for v in III IV; do echo "$v $(timeout 300 $B --config box2d9p_10240 --s2r-variant $v 2>/dev/null)" >> $OUT/sweep.txt; done
