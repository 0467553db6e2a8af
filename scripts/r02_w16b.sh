#!/bin/bash
OUT=gpurun_out/r02w16b; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_coverage.py -q -k "3d or star3d or heat3d" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --config star3d13p_512 > $OUT/bench.jsonl 2>>$OUT/err.txt
