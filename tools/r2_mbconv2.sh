#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/parity_errors.jsonl
timeout 900 python -m pytest tests/test_gpu_mbconv.py -q -m gpu -x -k pattern > gpurun_out/pytest_mbconv.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_mbconv.txt
timeout 1500 python tools/ablation_mbconv.py gpurun_out/mbconv_ablation.jsonl > gpurun_out/mbconv_ablation.log 2>&1
echo done
