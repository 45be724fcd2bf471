#!/bin/bash
# Swin LN rows: several rows per warp (default) vs one (SOUFFLE_SWIN_LN_RPW1=1): parity + traces
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_swin.py -q -m gpu -x > gpurun_out/pytest_swin.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_swin.txt
for b in 1 64; do
  timeout 300 python tools/swin_trace.py $b > gpurun_out/swl_b$b.txt 2>&1
  SOUFFLE_SWIN_LN_RPW1=1 timeout 300 python tools/swin_trace.py $b > gpurun_out/sw1r_b$b.txt 2>&1
done
echo done
