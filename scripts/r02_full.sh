#!/bin/bash
# round 2: whole GPU suite, smoke, bench over every config, launch list, dmma counters
OUT=gpurun_out/r02o; mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > $OUT/gpu_all.log 2>&1; echo "rc=$?" >> $OUT/gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
for c in box2d9p_10240 heat2d_10240 star2d9p_10240 box2d25p_10240 star2d13p_10240 box2d49p_10240 star2d13p_10240_tf2 box2d49p_10240_tf2 heat3d_512 box3d27p_512 star3d13p_512 box3d125p_512 star3d19p_512 box3d343p_512 heat1d_10240000 1d5p_10240000 heat1d_102400000 1d5p_102400000 heat1d_1024; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline >> $OUT/bench_all.jsonl 2>> $OUT/bench.err || echo "{\"config\": \"$c\", \"error\": true}" >> $OUT/bench_all.jsonl
done
for c in box2d9p_10240 box2d49p_10240 heat3d_512 box3d27p_512 heat1d_10240000; do
  timeout 900 python bench.py --config $c --engine tc_s2r --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator >> $OUT/bench_s2r.jsonl 2>> $OUT/bench.err
done
timeout 900 python bench.py --steps 5 --warmup 3 > $OUT/bench_default.json 2>> $OUT/bench.err
/usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $OUT/launches_box2d9p.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-comparator > /dev/null 2>&1
timeout 2400 python scripts/dmma_counters.py --out $OUT/dmma.json > $OUT/dmma.log 2>&1
