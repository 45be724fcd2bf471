#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/parity_errors.jsonl
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_swin.py -q -m gpu -x -k "rowwise or tensor_cache or random or tiny or fig2" > gpurun_out/pytest_reuse.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_reuse.txt
REUSE_SWEEP=1 timeout 900 python tools/reuse_effect.py > gpurun_out/reuse_effect.jsonl 2> gpurun_out/reuse_effect.err
echo done
