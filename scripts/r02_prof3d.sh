#!/bin/bash
# ncu --set full with source of the 3D kernels (Heat-3D tb2 / Tf=1, Box-3D27P, Star-3D13P): SASS stall maps
OUT=gpurun_out/r02p; mkdir -p $OUT
NCU=/usr/local/cuda/bin/ncu
cap() {
  local name=$1 kre=$2; shift 2
  timeout 900 $NCU --set full --clock-control none --import-source on -k regex:$kre -s 2 -c 1 -o $OUT/$name -f python scripts/one_run.py "$@" > /dev/null 2>&1
  $NCU -i $OUT/$name.ncu-rep --page source --csv --print-source sass > $OUT/${name}_sass.csv 2>/dev/null
  python scripts/ncu_brief.py $OUT/$name.ncu-rep > $OUT/${name}_brief.txt 2>&1
  $NCU -i $OUT/$name.ncu-rep --page raw --csv > $OUT/${name}_raw.csv 2>/dev/null
  rm -f $OUT/$name.ncu-rep
}
cap heat3d_tb2 k_tile3d_tb2 --config heat3d_512 --T 12
cap heat3d_tf1 k_tile3d --config heat3d_512 --T 6 --fuse 1
cap box3d27p k_tile3d --config box3d27p_512 --T 6
cap star3d13p k_tile3d --config star3d13p_512 --T 6
