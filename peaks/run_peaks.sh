#!/bin/bash
# Runs the FP64 peak microbenchmarks on the GPU box with an nvidia-smi clock record beside them.
set -e
cd "$(dirname "$0")"
mkdir -p ../gpurun_out
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap --format=csv -lms 200 > ../gpurun_out/peaks_clocks.csv &
SMI=$!
./fp64_peaks > ../gpurun_out/peaks_fp64.json
kill $SMI
cat ../gpurun_out/peaks_fp64.json
