#!/bin/bash
# ResNeXt blocks: GPU parity (generic executor) + Table 4 ladder timings
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_resnext.py -q -m gpu > gpurun_out/pytest_resnext.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_resnext.txt
timeout 1500 python tools/ablation_resnext.py gpurun_out/r02_resnext_ablation.jsonl > gpurun_out/resnext_ablation.log 2>&1
echo done
