#!/bin/bash
mkdir -p gpurun_out
for i in 0 3 9; do timeout 300 python tools/profile_generic.py mbconv:$i > gpurun_out/mbprof_$i.txt 2>&1; done
echo done
