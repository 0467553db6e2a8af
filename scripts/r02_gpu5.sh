#!/bin/bash
OUT=gpurun_out/r02e; mkdir -p $OUT
timeout 300 python scripts/dbg_wf.py > $OUT/dbg_wf.txt 2>&1
cuobjdump -sass -fun '_ZN3csx13k_direct2d_wfILi1ELi1ELi2ELi256ELi1EEEvNS_10DirectArgsENS_9WFWeightsE' paper_conf_ppopp_chenlwbwmyzcy24_b200/libcsx.so > $OUT/sass_wf111.txt 2>&1
