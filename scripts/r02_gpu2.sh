#!/bin/bash
# round 2, second GPU call: teardown tests, DMMA counters for every config, bench lines
OUT=gpurun_out/r02b; mkdir -p $OUT
timeout 600 python -m pytest tests/test_gpu_coverage.py -q -k "teardown" > $OUT/teardown.log 2>&1; echo "rc=$?" >> $OUT/teardown.log
timeout 1800 python scripts/dmma_counters.py --out $OUT/dmma.json > $OUT/dmma.log 2>&1
for c in box2d9p_10240 heat1d_10240000 heat1d_102400000 1d5p_102400000 heat3d_512 box3d27p_512 box3d125p_512 star3d13p_512 box3d343p_512 star3d19p_512; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline >> $OUT/bench.jsonl 2>> $OUT/bench.err
done
for c in box3d125p_512 box3d343p_512; do
  timeout 600 python bench.py --config $c --engine direct --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator >> $OUT/bench_direct.jsonl 2>> $OUT/bench.err
done
