#!/bin/bash
# MMoE: parity, graph-replay device time of the cluster kernel vs the single-CTA kernel
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k mmoe > gpurun_out/pytest_mmoe.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_mmoe.txt
for i in 1 2; do timeout 300 python tools/graph_timing.py > gpurun_out/gt_cluster_$i.json 2>&1; done
for i in 1 2; do SOUFFLE_MMOE_SINGLE=1 timeout 300 python tools/graph_timing.py > gpurun_out/gt_single_$i.json 2>&1; done
echo done
