#!/bin/bash
mkdir -p gpurun_out
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
timeout 600 python bench.py --swin-child 0 > gpurun_out/swin_child.json 2> gpurun_out/swin_child.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/swin_launches_b64.csv python tools/run_swin_once.py 64 2 > gpurun_out/ncu_swin_l.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/swin_launches_b1.csv python tools/run_swin_once.py 1 2 > gpurun_out/ncu_swin_l1.log 2>&1
timeout 900 python -m pytest tests/test_gpu_bert_stages.py -q -m gpu -k ffn1 > gpurun_out/pytest_ffn1.txt 2>&1
echo done
