#!/bin/bash
# full GPU suite (achieved errors logged) + graph-replay timings
mkdir -p gpurun_out
rm -f gpurun_out/parity_errors.jsonl
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/suite_pytest_gpu.txt 2>&1
echo "rc=$?" >> gpurun_out/suite_pytest_gpu.txt
timeout 300 python tools/graph_timing.py > gpurun_out/suite_graph_timing.json 2>&1
echo done
