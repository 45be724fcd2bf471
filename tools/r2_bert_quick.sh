#!/bin/bash
# BERT kernel change check: BERT GPU tests, bench line (no extras), stage timeline
mkdir -p gpurun_out
timeout 900 python -m pytest tests -q -m gpu -x -k "bert" > gpurun_out/q_pytest_bert.txt 2>&1
echo "rc=$?" >> gpurun_out/q_pytest_bert.txt
timeout 600 python bench.py --no-cpu-baseline --no-v0 --no-models > gpurun_out/q_bench.json 2> gpurun_out/q_bench.err
timeout 300 python tools/profile_bert.py 12 > gpurun_out/q_timeline.txt 2>&1
echo done
