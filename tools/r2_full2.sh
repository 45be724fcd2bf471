#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/parity_errors.jsonl
python -c "import __graft_entry__ as e; e.build()" > gpurun_out/build.log 2>&1
timeout 600 python -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/r02_smoke.txt 2>&1
echo "rc=$?" >> gpurun_out/r02_smoke.txt
timeout 1800 python -m pytest tests -q -m gpu > gpurun_out/r02_pytest_gpu.txt 2>&1
echo "rc=$?" >> gpurun_out/r02_pytest_gpu.txt
SOUFFLE_LSTM_PROF_CTA=75 timeout 300 python tools/profile_lstm.py > gpurun_out/lstm_timeline.txt 2>&1
timeout 1800 python bench.py > gpurun_out/r02_bench.json 2> gpurun_out/r02_bench.err
echo done
