#!/bin/bash
# BERT A/B timing: default vs SOUFFLE_BERT_DBG_SKIP=$AB_BITS (alternating, 3 rounds each) + parity
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bert_stages.py tests/test_gpu_parity.py -q -m gpu -k "bert" > gpurun_out/pytest_bert.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_bert.txt
rm -f gpurun_out/ab.txt
for i in 1 2 3; do
  timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-v0 --no-models 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('new', d['ms_per_step'])" >> gpurun_out/ab.txt
  SOUFFLE_BERT_DBG_SKIP=$AB_BITS timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-v0 --no-models 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('old', d['ms_per_step'])" >> gpurun_out/ab.txt
done
echo done
