#!/bin/bash
# BERT: parity (pattern kernel tests) + stage timeline
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bert_stages.py tests/test_gpu_parity.py -q -m gpu -k "bert" > gpurun_out/pytest_bert.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_bert.txt
timeout 300 python tools/profile_bert.py 12 > gpurun_out/bert_tl_base.txt 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-v0 --no-models > gpurun_out/bench_quick.json 2> gpurun_out/bench_quick.err
echo done
