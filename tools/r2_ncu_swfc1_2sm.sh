#!/bin/bash
# ncu --set full of the same FC1 GEMM on the 2-SM (cta_group::2) kernel
mkdir -p gpurun_out
SOUFFLE_SWIN_2SM=1 timeout 900 ncu --set full --import-source on --clock-control none -k regex:sw_gemm -s 21 -c 1 -o gpurun_out/ncu_swfc1_2sm python tools/run_swin_once.py 64 1 > gpurun_out/ncu_swfc1_2sm.log 2>&1
echo done
