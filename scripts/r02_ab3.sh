#!/bin/bash
cp scratch_so/libcsx_cur3.so paper_conf_ppopp_chenlwbwmyzcy24_b200/libcsx.so
OUT=gpurun_out/r02ab3; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_coverage.py -q -k "3d or star3d" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
CSX_TB_GEOM=7 timeout 300 python scripts/tb2_parity.py >> $OUT/t.log 2>&1
bash scripts/r02_ab_so.sh $OUT/heat prev cur3 -- --config heat3d_512
CSX_TB_GEOM=7 bash scripts/r02_ab_so.sh $OUT/heat7 prev cur3 -- --config heat3d_512
bash scripts/r02_ab_so.sh $OUT/box prev cur3 -- --config box3d27p_512
bash scripts/r02_ab_so.sh $OUT/s13 prev cur3 -- --config star3d13p_512
cp scratch_so/libcsx_cur3.so paper_conf_ppopp_chenlwbwmyzcy24_b200/libcsx.so
