#!/bin/bash
OUT=gpurun_out/r02d; mkdir -p $OUT
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py -q -k "1d or tile1d or heat1d or 1d5p" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
for c in heat1d_102400000 1d5p_102400000 heat1d_10240000 1d5p_10240000; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --config $c >> $OUT/bench.jsonl 2>>$OUT/err.txt
done
