#!/bin/bash
# On the GPU box: the ncu evidence committed under profiles/ (round tag $1).
#   launches_<cfg>.csv : every launch of a short bench run (gpu__time_duration, cold, serialised)
#   prof_<kernel>.ncu-rep : one `ncu --set full` capture of the dominant kernel per engine/config
TAG=${1:-r01}
mkdir -p gpurun_out/$TAG
NCU=/usr/local/cuda/bin/ncu
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-comparator"
$NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
     --log-file gpurun_out/$TAG/launches_box2d9p_tc_tile.csv $B > /dev/null 2>&1
cap() {  # name kernel-regex skip bench-args...
  local name=$1 kre=$2 skip=$3; shift 3
  $NCU --set full --clock-control none --import-source on -k regex:$kre -s $skip -c 1 \
       -o gpurun_out/$TAG/prof_$name -f python bench.py --steps 1 --warmup 3 --no-e2e \
       --no-cpu-baseline --no-comparator "$@" > gpurun_out/$TAG/prof_$name.log 2>&1
}
cap box2d9p_tc_tile k_tile2d 3
cap box2d9p_tc_s2r k_s2r2d 3 --engine tc_s2r
cap box2d9p_direct k_direct2d 3 --engine direct
cap box3d27p_tc_tile k_tile3d 3 --config box3d27p_512
cap heat3d_tc_tile k_tile3d 3 --config heat3d_512
cap heat1d_tc_tile k_tile1d 5 --config heat1d_10240000
cap box2d49p_tc_tile k_tile2d 3 --config box2d49p_10240
cap box2d49p_tf2_tc_tile k_tile2d 3 --config box2d49p_10240_tf2
cap 1d5p_tc_tile k_tile1d 5 --config 1d5p_10240000
ls -la gpurun_out/$TAG
