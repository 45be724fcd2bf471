#!/bin/bash
# One GPU call: bench (default config), ncu launch list of the bench, ncu --set full of the BERT and
# LSTM kernels.  Outputs land in gpurun_out/ (summarised into profiles/ by tools/ncu_summary.py).
mkdir -p gpurun_out
nvidia-smi > gpurun_out/nvsmi.txt 2>&1
timeout 900 python bench.py > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-v0 --no-models > gpurun_out/ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bert_kernel -s 1 -c 1 -o gpurun_out/prof_bert python tools/run_once.py bert_base 0 0 2 > gpurun_out/ncu_full.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:lstm_kernel -s 1 -c 1 -o gpurun_out/prof_lstm python tools/profile_lstm.py > gpurun_out/ncu_lstm.log 2>&1
echo done
