#!/bin/bash
# MMoE kernel device time: ncu launch list with warm caches (graph-like steady state) and cold caches
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:mmoe_kernel -s 20 -c 20 --csv python tools/mmoe_timing.py > gpurun_out/ncu_mmoe_warm.csv 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control all -k regex:mmoe_kernel -s 20 -c 20 --csv python tools/mmoe_timing.py > gpurun_out/ncu_mmoe_cold.csv 2>&1
echo done
