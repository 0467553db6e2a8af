#!/bin/bash
# A/B of two builds of libcsx.so (scratch_so/libcsx_<tag>.so) on one config: usage r02_ab_so.sh OUT tagA tagB -- bench args
OUT=$1; A=$2; B=$3; shift 4
mkdir -p $OUT
LIB=paper_conf_ppopp_chenlwbwmyzcy24_b200/libcsx.so
for rep in 1 2; do for t in $A $B; do
  cp scratch_so/libcsx_$t.so $LIB
  echo "$t $(timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-comparator "$@" 2>/dev/null)" >> $OUT/ab.txt
done; done
