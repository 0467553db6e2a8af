#!/bin/bash
# 2D r = 1 TC_TILE auto depth 2: parity, DMMA counters of the new dominant kernel, bench lines
OUT=gpurun_out/r02tf2; mkdir -p $OUT
cp profiles/dmma_counters.json $OUT/dmma.json
timeout 900 python scripts/dmma_counters.py --out $OUT/dmma.json box2d9p_10240:tc_tile heat2d_10240:tc_tile > $OUT/dmma.log 2>&1
cp $OUT/dmma.json profiles/dmma_counters.json
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_coverage.py -q -k "full_extent_parity and box2d9p or run_host or 2d or wrap" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
timeout 900 python bench.py --steps 5 --warmup 3 > $OUT/bench_default.json 2>> $OUT/err.txt
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --config heat2d_10240 > $OUT/bench_heat2d.json 2>> $OUT/err.txt
timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --engine tc_s2r > $OUT/bench_s2r.json 2>> $OUT/err.txt
