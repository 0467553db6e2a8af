#!/bin/bash
OUT=gpurun_out/r02l; mkdir -p $OUT
NCU=/usr/local/cuda/bin/ncu
for c in star3d13p_512 heat3d_512 box3d27p_512; do
  $NCU --set full --clock-control none --import-source on -k regex:k_tile3d -s 2 -c 1 -o $OUT/prof_$c -f python scripts/one_run.py --config $c --T 6 > $OUT/prof_$c.log 2>&1
  python scripts/ncu_brief.py $OUT/prof_$c.ncu-rep > $OUT/brief_$c.txt 2>&1
  $NCU -i $OUT/prof_$c.ncu-rep --page source --csv > $OUT/src_$c.csv 2>/dev/null
done
mkdir -p /tmp/reps; mv $OUT/*.ncu-rep /tmp/reps/
