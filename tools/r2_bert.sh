#!/bin/bash
mkdir -p gpurun_out
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_bert_stages.py tests/test_gpu_parity.py -q -x -m gpu -k "bert or stage or layernorm or bias" > gpurun_out/pytest_bert.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_bert.txt
timeout 300 python tools/sweep_bert.py "" > gpurun_out/sweep_now.txt 2>&1
timeout 300 python tools/profile_bert.py 12 > gpurun_out/timeline.txt 2>&1
echo done
