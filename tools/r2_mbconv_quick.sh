#!/bin/bash
# MBConv pattern: parity + per-block latency (pattern vs unfused) through the bench helper
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_mbconv.py -q -m gpu -x > gpurun_out/pytest_mbconv.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_mbconv.txt
timeout 1500 python tools/ablation_mbconv.py gpurun_out/mbconv_ablation.jsonl > gpurun_out/mbconv_ablation.log 2>&1
echo done
