#!/bin/bash
mkdir -p gpurun_out
timeout 600 ncu --set full --import-source on --clock-control none -k regex:lstm_kernel -c 1 -o gpurun_out/ncu_lstm_full python tools/profile_lstm.py > gpurun_out/ncu_lstm_full.log 2>&1
echo "rc=$?" >> gpurun_out/ncu_lstm_full.log
echo done
