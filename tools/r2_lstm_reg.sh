#!/bin/bash
# LSTM register-resident GEMV: parity, timeline, graph-replay latency, A/B against the smem kernel
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k lstm > gpurun_out/pytest_lstm.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_lstm.txt
SOUFFLE_LSTM_PROF_CTA=75 timeout 300 python tools/profile_lstm.py > gpurun_out/lstm_timeline_reg.txt 2>&1
SOUFFLE_LSTM_SMEM=1 SOUFFLE_LSTM_PROF_CTA=75 timeout 300 python tools/profile_lstm.py > gpurun_out/lstm_timeline_smem.txt 2>&1
for i in 1 2; do timeout 300 python tools/graph_timing.py > gpurun_out/graph_timing_reg_$i.json 2>&1; done
SOUFFLE_LSTM_SMEM=1 timeout 300 python tools/graph_timing.py > gpurun_out/graph_timing_smem.json 2>&1
echo done
