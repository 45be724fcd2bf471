#!/bin/bash
mkdir -p gpurun_out
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bert_stages.py tests/test_gpu_swin.py -q -m gpu > gpurun_out/pytest_mix.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_mix.txt
SOUFFLE_MMOE_DEBUG=1 timeout 120 python tools/mmoe_timing.py > gpurun_out/mmoe_dbg.txt 2>&1
timeout 300 python tools/graph_timing.py > gpurun_out/graph_timing.json 2> gpurun_out/graph_timing.err
timeout 300 python tools/sweep_bert.py "" > gpurun_out/sweep_now.txt 2>&1
timeout 600 python bench.py --swin-child 0 > gpurun_out/swin_child.json 2> gpurun_out/swin_child.err
timeout 300 python tools/swin_trace.py 64 > gpurun_out/trace_b64.txt 2>&1
echo done
