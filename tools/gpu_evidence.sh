#!/bin/bash
# One GPU call collecting the round's evidence into gpurun_out/ (summarised into profiles/ by
# tools/ncu_summary.py): GPU tests, the default bench line, the ncu launch list of a short bench run,
# and ncu --set full captures of the BERT and LSTM kernels and of the first Swin-B launch.
mkdir -p gpurun_out
nvidia-smi > gpurun_out/nvsmi.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.txt 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.txt
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?" >> gpurun_out/bench.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-v0 --no-models > gpurun_out/ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bert_kernel -s 1 -c 1 \
  -o gpurun_out/prof_bert -f python tools/run_model_once.py bert 2 > gpurun_out/ncu_bert.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:lstm_kernel -s 1 -c 1 \
  -o gpurun_out/prof_lstm -f python tools/run_model_once.py lstm 2 > gpurun_out/ncu_lstm.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:souffle_exec_kernel -s 7 -c 1 \
  -o gpurun_out/prof_swin -f python tools/run_model_once.py swin 2 > gpurun_out/ncu_swin.log 2>&1
echo done
