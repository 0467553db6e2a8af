#!/bin/bash
bash scripts/r02_ab_so.sh gpurun_out/r02ab2/box prev cur -- --config box3d27p_512
bash scripts/r02_ab_so.sh gpurun_out/r02ab2/heat prev cur -- --config heat3d_512
bash scripts/r02_ab_so.sh gpurun_out/r02ab2/heat1 prev cur -- --config heat3d_512 --fuse 1
bash scripts/r02_ab_so.sh gpurun_out/r02ab2/c2 prev cur -- --config box2d9p_10240
cp scratch_so/libcsx_cur.so paper_conf_ppopp_chenlwbwmyzcy24_b200/libcsx.so
