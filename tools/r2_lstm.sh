#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k lstm > gpurun_out/pytest_lstm.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_lstm.txt
SOUFFLE_LSTM_SIMT=1 timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k lstm >> gpurun_out/pytest_lstm.txt 2>&1
echo "rc_simt=$?" >> gpurun_out/pytest_lstm.txt
SOUFFLE_LSTM_PROF_CTA=75 timeout 300 python tools/profile_lstm.py > gpurun_out/lstm_timeline.txt 2>&1
SOUFFLE_LSTM_SIMT=1 SOUFFLE_LSTM_PROF_CTA=75 timeout 300 python tools/profile_lstm.py > gpurun_out/lstm_timeline_simt.txt 2>&1
timeout 300 python tools/graph_timing.py > gpurun_out/graph_timing.json 2>&1
echo done
