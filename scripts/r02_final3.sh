#!/bin/bash
# round 2 closing pass: GPU suite, smoke, bench over every config (e2e through the chunked
# csx_run_host), default bench, e2e chunk-count sweep on C2
OUT=gpurun_out/r02h3; mkdir -p $OUT
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > $OUT/gpu_all.log 2>&1; echo "rc=$?" >> $OUT/gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
for c in box2d9p_10240 heat2d_10240 star2d9p_10240 box2d25p_10240 star2d13p_10240 box2d49p_10240 star2d13p_10240_tf2 box2d49p_10240_tf2 heat3d_512 box3d27p_512 star3d13p_512 box3d125p_512 star3d19p_512 box3d343p_512 heat1d_10240000 1d5p_10240000 heat1d_102400000 1d5p_102400000 heat1d_1024; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline >> $OUT/bench_all.jsonl 2>> $OUT/bench.err || echo "{\"config\": \"$c\", \"error\": true}" >> $OUT/bench_all.jsonl
done
timeout 900 python bench.py --steps 5 --warmup 3 > $OUT/bench_default.json 2>> $OUT/bench.err
for k in 4 8 12 16; do echo "chunks=$k $(CSX_HOST_CHUNKS=$k timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-comparator 2>/dev/null)" >> $OUT/e2e_chunks.txt; done
