#!/bin/bash
mkdir -p gpurun_out
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k lstm > gpurun_out/pytest_lstm.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_lstm.txt
SOUFFLE_LSTM_PROF_CTA=75 timeout 300 python tools/profile_lstm.py > gpurun_out/lstm_timeline.txt 2>&1
timeout 300 python tools/graph_timing.py > gpurun_out/graph_timing.json 2>&1
echo done
