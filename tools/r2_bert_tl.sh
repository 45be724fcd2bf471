#!/bin/bash
# BERT: stage-isolation / parity tests, sub-stage timeline, quick bench
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bert_stages.py tests/test_gpu_parity.py -q -m gpu -k "bert" > gpurun_out/pytest_bert.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_bert.txt
timeout 300 python tools/profile_bert.py 12 > gpurun_out/bert_tl_base.txt 2>&1
for i in 1 2; do timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-v0 --no-models 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('bench', d['ms_per_step'])" >> gpurun_out/bert_tl_base.txt; done
echo done
