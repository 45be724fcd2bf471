#!/bin/bash
# Swin: parity + traces b1 / b8 / b64 (current build)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_swin.py -q -m gpu -x > gpurun_out/pytest_swin.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_swin.txt
for b in 1 8 64; do timeout 300 python tools/swin_trace.py $b > gpurun_out/swq_b$b.txt 2>&1; done
echo done
