#!/bin/bash
# compute-sanitizer (racecheck / synccheck / memcheck) on the kernels changed late in round 2: the
# register-resident LSTM kernel, the MMoE cluster kernel, the Swin GEMM staged epilogues, the BERT kernel
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for c in lstm_small mmoe swin_small bert_small; do
  for tool in racecheck synccheck memcheck; do
    timeout 900 $CS --tool $tool python tools/san_case.py $c > gpurun_out/san_${tool}_$c.txt 2>&1
  done
done
echo done
