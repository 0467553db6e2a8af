#!/bin/bash
OUT=gpurun_out/r02last2; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py -q -k "1d or tile1d or heat1d or 1d5p" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-comparator"
for c in heat1d_102400000 1d5p_102400000 heat1d_10240000 1d5p_10240000; do timeout 600 $B --config $c >> $OUT/bench.jsonl 2>>$OUT/err.txt; done
