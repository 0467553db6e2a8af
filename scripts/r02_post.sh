#!/bin/bash
OUT=gpurun_out/r02post; mkdir -p $OUT
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py -q -k "run_host or tile_variants or 16_warps or general_radius_variants" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
timeout 600 python bench.py --steps 5 --warmup 3 > $OUT/bench_default.json 2>> $OUT/err.txt
for c in heat3d_512 heat1d_102400000 box3d27p_512; do timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-comparator --config $c >> $OUT/bench_e2e.jsonl 2>> $OUT/err.txt; done
bash scripts/r02_s19.sh
