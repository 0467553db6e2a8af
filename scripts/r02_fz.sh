#!/bin/bash
bash scripts/r02_ab_so.sh gpurun_out/r02fz fz0 fz1 -- --config heat3d_512
CSX_TB_GEOM=3 bash scripts/r02_ab_so.sh gpurun_out/r02fz3 fz0 fz1 -- --config heat3d_512
cp scratch_so/libcsx_fz0.so paper_conf_ppopp_chenlwbwmyzcy24_b200/libcsx.so
for v in 0 i j; do echo "v=$v $(CSX_TILE3D_VARIANT=$v timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator --config box3d27p_512 2>/dev/null)" >> gpurun_out/r02fz/box.txt; done
