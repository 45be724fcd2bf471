#!/bin/bash
mkdir -p gpurun_out
for i in 1 2 3; do timeout 300 python tools/swin_trace.py 64 > gpurun_out/swtrace_b64_$i.txt 2>&1; done
echo done
