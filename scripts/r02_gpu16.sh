#!/bin/bash
OUT=gpurun_out/r02u; mkdir -p $OUT
/usr/local/cuda/bin/ncu --set full --import-source on --clock-control none -k regex:k_tile3d_tb2 -s 2 -c 1 -o $OUT/prof_tb2 -f python scripts/one_run.py --config heat3d_512 --T 12 --fuse 2 > /dev/null 2>&1
/usr/local/cuda/bin/ncu -i $OUT/prof_tb2.ncu-rep --page source --csv --print-source sass > $OUT/src_sass.csv 2>&1
/usr/local/cuda/bin/ncu -i $OUT/prof_tb2.ncu-rep --page source --csv --print-source cuda > $OUT/src_cuda.csv 2>&1
rm -f $OUT/prof_tb2.ncu-rep
