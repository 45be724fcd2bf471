#!/bin/bash
mkdir -p gpurun_out
rm -f gpurun_out/ab.txt
for i in 1 2 3; do
  timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-v0 --no-models 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('base', d['ms_per_step'])" >> gpurun_out/ab.txt
  SOUFFLE_BERT_DBG_SKIP=$AB_BITS timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-v0 --no-models 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('exp', d['ms_per_step'])" >> gpurun_out/ab.txt
done
SOUFFLE_BERT_DBG_SKIP=$AB_BITS timeout 300 python tools/profile_bert.py 12 > gpurun_out/bert_tl_exp.txt 2>&1
echo done
