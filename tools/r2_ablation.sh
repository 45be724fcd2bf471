#!/bin/bash
mkdir -p gpurun_out
timeout 1800 python tools/ablation.py mmoe bert lstm swin > gpurun_out/ablation.jsonl 2> gpurun_out/ablation.err
echo done
