#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/parity_errors.jsonl
timeout 1500 python -m pytest tests -q -m gpu -x > gpurun_out/pytest_gpu.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_gpu.txt
timeout 900 python tools/reuse_effect.py > gpurun_out/reuse_effect.jsonl 2> gpurun_out/reuse_effect.err
echo done
