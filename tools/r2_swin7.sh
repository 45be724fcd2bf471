#!/bin/bash
mkdir -p gpurun_out
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
timeout 300 python -m pytest tests/test_gpu_swin.py -q -m gpu -k "pattern" > gpurun_out/pytest_swin.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_swin.txt
timeout 600 python bench.py --swin-child 0 > gpurun_out/swin_child.json 2> gpurun_out/swin_child.err
SOUFFLE_SWIN_2SM=0 timeout 300 python tools/swin_trace.py 64 > gpurun_out/trace_b64_1sm.txt 2>&1
timeout 300 python tools/swin_trace.py 64 > gpurun_out/trace_b64.txt 2>&1
echo done
