#!/bin/bash
# ncu --set full of the Swin-B b64 stage-3 block-0 FC1 GEMM (22nd sw_gemm launch), packed-GELU epilogue
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:sw_gemm -s 21 -c 1 -o gpurun_out/ncu_swfc1_r2b python tools/run_swin_once.py 64 1 > gpurun_out/ncu_swfc1_r2b.log 2>&1
echo done
