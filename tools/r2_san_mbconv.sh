#!/bin/bash
# compute-sanitizer on the MBConv pattern kernel (expand 1 / 6, kernel 3 / 5, stride 1 / 2, split-K project)
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for i in 0 1 9; do
  for tool in racecheck synccheck memcheck; do
    timeout 900 $CS --tool $tool python tools/san_case.py mbconv:$i > gpurun_out/san_${tool}_mbconv$i.txt 2>&1
  done
done
echo done
