#!/bin/bash
# HEAD verification: GPU suite, smoke, default bench line
OUT=gpurun_out/r02v; mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q > $OUT/gpu_all.log 2>&1; echo "rc=$?" >> $OUT/gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench_default.json 2>> $OUT/err.txt
