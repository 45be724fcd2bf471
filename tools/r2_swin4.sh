#!/bin/bash
mkdir -p gpurun_out
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
timeout 300 python -m pytest tests/test_gpu_swin.py -q -x -m gpu -k "pattern_small or generic_agree" > gpurun_out/pytest_swin.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_swin.txt
SOUFFLE_SWIN_2SM=1 timeout 300 python tools/swin_trace.py 64 > gpurun_out/trace_b64_2sm.txt 2>&1
SOUFFLE_SWIN_2SM=1 timeout 600 python -m pytest tests/test_gpu_swin.py -q -x -m gpu -k "full_size" > gpurun_out/pytest_swin_full.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_swin_full.txt
echo done
