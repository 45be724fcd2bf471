#!/bin/bash
# ResNeXt pattern: parity + phase timeline
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_resnext.py -q -m gpu -k pattern > gpurun_out/pytest_resnext.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_resnext.txt
timeout 600 python tools/profile_resnext.py > gpurun_out/rx_prof.txt 2>&1
echo done
