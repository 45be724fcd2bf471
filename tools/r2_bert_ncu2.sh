#!/bin/bash
mkdir -p gpurun_out
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_bert_stages.py tests/test_gpu_parity.py -q -x -m gpu -k "bert or stage or layernorm or bias" > gpurun_out/pytest_bert.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_bert.txt
timeout 300 python tools/sweep_bert.py "" > gpurun_out/sweep_now.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-v0 --no-models > gpurun_out/r02_ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bert_kernel -s 1 -c 1 -o gpurun_out/r02_prof_bert python tools/run_once.py bert_base 0 0 2 > gpurun_out/r02_ncu_full.log 2>&1
SOUFFLE_LSTM_PROF_CTA=75 timeout 300 python tools/profile_lstm.py > gpurun_out/lstm_timeline.txt 2>&1
echo done
