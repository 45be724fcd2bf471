#!/bin/bash
# MMoE: parity, per-phase clocks (debug printf), graph-replay device time
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k mmoe > gpurun_out/pytest_mmoe.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_mmoe.txt
SOUFFLE_MMOE_DEBUG=1 timeout 300 python tools/mmoe_timing.py > gpurun_out/mmoe_dbg.txt 2>&1
for i in 1 2; do timeout 300 python tools/graph_timing.py > gpurun_out/graph_timing_$i.json 2>&1; done
echo done
