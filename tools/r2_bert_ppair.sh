#!/bin/bash
# BERT pair-reduced partials: BERT GPU tests, A/B bench (default vs SOUFFLE_BERT_PPAIR=0), timeline
mkdir -p gpurun_out
rm -f gpurun_out/ab.txt
timeout 900 python -m pytest tests -q -m gpu -x -k "bert" > gpurun_out/q_pytest_bert.txt 2>&1
echo "rc=$?" >> gpurun_out/q_pytest_bert.txt
for i in 1 2 3; do
  timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-v0 --no-models 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('ppair', d['latency_us_median'])" >> gpurun_out/ab.txt
  SOUFFLE_BERT_PPAIR=0 timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-v0 --no-models 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('base', d['latency_us_median'])" >> gpurun_out/ab.txt
done
timeout 300 python tools/profile_bert.py 12 > gpurun_out/q_timeline.txt 2>&1
echo done
