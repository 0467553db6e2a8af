#!/bin/bash
# round 2 re-entry: HEAD verification (GPU suite, smoke, default bench, reference arm, bench lines)
OUT=gpurun_out/r02h; mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q --durations=15 > $OUT/gpu_all.log 2>&1; echo "rc=$?" >> $OUT/gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
timeout 900 python bench.py --steps 5 --warmup 3 > $OUT/bench_default.json 2>> $OUT/bench.err
for c in heat3d_512 box3d27p_512 heat1d_102400000 1d5p_102400000 heat1d_10240000; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline >> $OUT/bench_lines.jsonl 2>> $OUT/bench.err
done
