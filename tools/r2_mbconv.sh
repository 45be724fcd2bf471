#!/bin/bash
# generic executor: parity of every generic-path suite, then the MBConv Fig. 5 variant latencies
mkdir -p gpurun_out
rm -f gpurun_out/parity_errors.jsonl
timeout 1800 python -m pytest tests/test_gpu_mbconv.py tests/test_gpu_parity.py tests/test_gpu_swin.py tests/test_gpu_se.py -q -m gpu -x > gpurun_out/pytest_mbconv.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_mbconv.txt
timeout 1500 python tools/ablation_mbconv.py gpurun_out/mbconv_ablation.jsonl > gpurun_out/mbconv_ablation.log 2>&1
echo done
