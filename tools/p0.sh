#!/bin/bash
# P0 box bring-up: FP64 peaks with clocks sampled during the run.
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap --format=csv -lms 200 > gpurun_out/p0_clocks.csv &
SMI=$!
./tools/fp64_peak > gpurun_out/p0_fp64.json
kill $SMI
nvidia-smi -q | head -40 > gpurun_out/p0_smi.txt
nproc > gpurun_out/p0_host.txt; lscpu | grep -i "model name" >> gpurun_out/p0_host.txt
cat gpurun_out/p0_fp64.json
