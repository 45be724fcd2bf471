#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_mbconv.py -q -m gpu -x -k pattern > gpurun_out/pytest_mbconv.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_mbconv.txt
timeout 600 python tools/profile_mbconv.py > gpurun_out/mbconv_phases.txt 2>&1
echo done
