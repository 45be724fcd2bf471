#!/bin/bash
# compute-sanitizer on the generic executor's row-block stages + tensor cache (default capacity and
# forced LRU spills)
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for case in rowwise swin_generic generic_tiny; do
  for tool in racecheck synccheck memcheck; do
    timeout 900 $CS --tool $tool python tools/san_case.py $case > gpurun_out/san_${tool}_${case}.txt 2>&1
    SOUFFLE_CACHE_FLOATS=2048 timeout 900 $CS --tool $tool python tools/san_case.py $case > gpurun_out/san_${tool}_${case}_spill.txt 2>&1
  done
done
echo done
