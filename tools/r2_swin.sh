#!/bin/bash
mkdir -p gpurun_out
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_swin.py -q -x -m gpu -k "pattern_small" > gpurun_out/pytest_swin.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_swin.txt
timeout 900 python -m pytest tests/test_gpu_bert_stages.py tests/test_gpu_swin.py -q -m gpu > gpurun_out/pytest_swin2.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_swin2.txt
echo done
