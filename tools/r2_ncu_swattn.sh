#!/bin/bash
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:sw_attn_kernel -s 4 -c 1 -o gpurun_out/ncu_swattn python tools/run_swin_once.py 64 1 > gpurun_out/ncu_swattn.log 2>&1
echo "rc=$?" >> gpurun_out/ncu_swattn.log
echo done
