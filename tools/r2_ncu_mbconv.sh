#!/bin/bash
mkdir -p gpurun_out
for i in 0 7; do
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:mbconv_kernel -s 1 -c 1 -o gpurun_out/ncu_mbconv_$i python tools/run_mbconv_once.py $i 2 > gpurun_out/ncu_mbconv_$i.log 2>&1
done
echo done
