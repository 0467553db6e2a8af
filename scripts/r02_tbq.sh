#!/bin/bash
OUT=gpurun_out/r02tbq; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_coverage.py tests/test_gpu_parity.py -q -k "tb2 or two_step or smoke or full_extent_parity and heat3d" > $OUT/t.log 2>&1; echo "rc=$?" >> $OUT/t.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "rc=$?" >> $OUT/smoke.log
