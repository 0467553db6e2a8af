#!/bin/bash
# round 2, first GPU call: new coverage tests, DMMA metric names, the whole GPU suite
OUT=gpurun_out/r02a; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $OUT/gpu.txt; nproc >> $OUT/gpu.txt
ncu --query-metrics > $OUT/metrics_all.txt 2>&1
grep -i "dmma\|fp64\|dp_\|tensor" $OUT/metrics_all.txt > $OUT/metrics_fp64.txt
timeout 1500 python -m pytest tests/test_gpu_coverage.py -q -k "not full_extent" -p no:randomly > $OUT/cov.log 2>&1; echo "cov rc=$?" >> $OUT/cov.log
timeout 1200 python -m pytest tests/test_gpu_coverage.py -q -k "full_extent" --durations=0 > $OUT/full.log 2>&1; echo "full rc=$?" >> $OUT/full.log
timeout 2400 python -m pytest tests -m gpu -q --deselect tests/test_gpu_coverage.py --durations=15 > $OUT/gpu_all.log 2>&1; echo "all rc=$?" >> $OUT/gpu_all.log
tail -3 $OUT/*.log
