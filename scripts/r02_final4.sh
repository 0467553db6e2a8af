#!/bin/bash
# round 2 closing pass at the final defaults (2D r = 1 TC_TILE Tf = 2, chunked csx_run_host)
OUT=gpurun_out/r02i; mkdir -p $OUT/brief
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > $OUT/gpu_all.log 2>&1; echo "rc=$?" >> $OUT/gpu_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
for c in box2d9p_10240 heat2d_10240 star2d9p_10240 box2d25p_10240 star2d13p_10240 box2d49p_10240 star2d13p_10240_tf2 box2d49p_10240_tf2 heat3d_512 box3d27p_512 star3d13p_512 box3d125p_512 star3d19p_512 box3d343p_512 heat1d_10240000 1d5p_10240000 heat1d_102400000 1d5p_102400000 heat1d_1024; do
  timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline >> $OUT/bench_all.jsonl 2>> $OUT/bench.err || echo "{\"config\": \"$c\", \"error\": true}" >> $OUT/bench_all.jsonl
done
timeout 900 python bench.py --config box2d9p_10240 --fuse 3 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator >> $OUT/bench_extra.jsonl 2>> $OUT/bench.err
timeout 900 python bench.py --config heat3d_512 --fuse 1 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator >> $OUT/bench_extra.jsonl 2>> $OUT/bench.err
for c in box2d9p_10240 box2d49p_10240 box2d25p_10240 box3d27p_512 heat1d_10240000 heat1d_102400000; do
  timeout 900 python bench.py --config $c --engine tc_s2r --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator >> $OUT/bench_s2r.jsonl 2>> $OUT/bench.err
done
timeout 900 python bench.py --steps 5 --warmup 3 > $OUT/bench_default.json 2>> $OUT/bench.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_reference.json 2>> $OUT/bench.err
NCU=/usr/local/cuda/bin/ncu
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $OUT/launches_box2d9p.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --no-comparator > /dev/null 2>&1
cap() {
  local name=$1 kre=$2 skip=$3; shift 3
  timeout 900 $NCU --set full --clock-control none --import-source on -k regex:$kre -s $skip -c 1 -o $OUT/prof_$name -f python scripts/one_run.py "$@" > /dev/null 2>&1
  python scripts/ncu_brief.py $OUT/prof_$name.ncu-rep > $OUT/brief/brief_$name.txt 2>&1
  $NCU -i $OUT/prof_$name.ncu-rep --page source --csv --print-source sass > $OUT/sass_$name.csv 2>/dev/null
  python scripts/sass_hot.py $OUT/sass_$name.csv 30 > $OUT/brief/sass_hot_$name.txt 2>&1
  rm -f $OUT/prof_$name.ncu-rep $OUT/sass_$name.csv
}
cap box2d9p_tc_tile k_tile2d 2 --config box2d9p_10240 --T 12
cap box3d343p_tc_tile k_tile3d 2 --config box3d343p_512 --T 4
