#!/bin/bash
# ncu --set full (source-level stall sampling) of the register-resident LSTM kernel
mkdir -p gpurun_out
timeout 600 ncu --set full --import-source on --clock-control none -k regex:lstm_reg_kernel -s 1 -c 1 -o gpurun_out/ncu_lstm_reg python tools/run_model_once.py lstm 3 > gpurun_out/ncu_lstm_reg.log 2>&1
echo "rc=$?" >> gpurun_out/ncu_lstm_reg.log
echo done
