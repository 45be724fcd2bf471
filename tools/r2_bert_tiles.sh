#!/bin/bash
# BERT pair-GEMM N-tile study (SOUFFLE_BERT_PAIR_NT=qkv,ffn1), alternating runs
mkdir -p gpurun_out
rm -f gpurun_out/tiles.txt
for i in 1 2; do
  for cfg in 32,64 64,64 32,32 64,32; do
    SOUFFLE_BERT_PAIR_NT=$cfg timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-v0 --no-models 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$cfg', d['ms_per_step'])" >> gpurun_out/tiles.txt
  done
done
SOUFFLE_BERT_PAIR_NT=64,64 timeout 600 python -m pytest tests/test_gpu_bert_stages.py tests/test_gpu_parity.py -q -m gpu -k "bert" > gpurun_out/pytest_bert.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_bert.txt
echo done
