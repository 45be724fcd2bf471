#!/bin/bash
# Swin b8 / b64 traces: 1-SM tiles (default) vs SOUFFLE_SWIN_2SM=1 (256 x 256 CTA-pair tiles)
mkdir -p gpurun_out
for b in 8 64; do
  timeout 300 python tools/swin_trace.py $b > gpurun_out/sw1_b$b.txt 2>&1
  SOUFFLE_SWIN_2SM=1 timeout 300 python tools/swin_trace.py $b > gpurun_out/sw2_b$b.txt 2>&1
done
SOUFFLE_SWIN_2SM=1 timeout 600 python -m pytest tests/test_gpu_swin.py -q -m gpu -k "b8 or b64 or 2sm" > gpurun_out/pytest_swin2.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_swin2.txt
echo done
