#!/bin/bash
# On the GPU box: launch list of one bench run and one `ncu --set full` capture of the dominant
# kernel.  Usage: scripts/profile.sh <tag> <kernel-regex> [bench args...]
set -x
TAG=$1; KRE=$2; shift 2
mkdir -p gpurun_out
NCU=/usr/local/cuda/bin/ncu
$NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
     --log-file gpurun_out/launches_${TAG}.csv \
     python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-comparator "$@" \
     > gpurun_out/launches_${TAG}.out 2>&1
$NCU --set full --clock-control none --import-source on -k regex:${KRE} -s 3 -c 1 \
     -o gpurun_out/prof_${TAG} -f \
     python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline --no-comparator "$@" \
     > gpurun_out/prof_${TAG}.out 2>&1
ls -la gpurun_out
