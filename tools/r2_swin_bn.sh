#!/bin/bash
# N-tile policy study of the Swin pattern GEMMs: in-graph launch traces at batch 1 / 8 / 64, new policy
# vs the previous one (SOUFFLE_SWIN_BN_OLD=1)
mkdir -p gpurun_out
for b in 1 8 64; do
  timeout 300 python tools/swin_trace.py $b > gpurun_out/swbn_new_b$b.txt 2>&1
  SOUFFLE_SWIN_BN_OLD=1 timeout 300 python tools/swin_trace.py $b > gpurun_out/swbn_old_b$b.txt 2>&1
done
timeout 600 python -m pytest tests/test_gpu_swin.py -q -m gpu > gpurun_out/pytest_swin.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_swin.txt
echo done
