#!/bin/bash
# evidence for the small models and sanitizers (round 2)
mkdir -p gpurun_out
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/bench_exchange tools/bench_exchange.cu
./tools/bench_exchange gpurun_out/exchange.json > gpurun_out/exchange.txt 2>&1
timeout 300 python tools/graph_timing.py > gpurun_out/graph_timing.json 2> gpurun_out/graph_timing.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:mmoe_kernel -c 20 --csv --log-file gpurun_out/ncu_mmoe.csv python tools/mmoe_timing.py > gpurun_out/ncu_mmoe.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active,sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,sm__inst_executed_pipe_fma.sum --clock-control none -k regex:lstm_kernel -s 1 -c 1 --csv --log-file gpurun_out/ncu_lstm_pipes.csv python tools/profile_lstm.py > gpurun_out/ncu_lstm2.log 2>&1
# sanitizers (small configs; every kernel family)
export PYTHONPATH=$PWD
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/san_case.py bert_small > gpurun_out/san_racecheck_bert.txt 2>&1
timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python tools/san_case.py bert_small > gpurun_out/san_synccheck_bert.txt 2>&1
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/san_case.py swin_small > gpurun_out/san_racecheck_swin.txt 2>&1
timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python tools/san_case.py swin_small > gpurun_out/san_synccheck_swin.txt 2>&1
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/san_case.py generic_tiny > gpurun_out/san_racecheck_generic.txt 2>&1
timeout 900 compute-sanitizer --tool synccheck --print-limit 20 python tools/san_case.py generic_tiny > gpurun_out/san_synccheck_generic.txt 2>&1
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python tools/san_case.py bert_small > gpurun_out/san_memcheck_bert.txt 2>&1
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python tools/san_case.py swin_small > gpurun_out/san_memcheck_swin.txt 2>&1
echo done
