#!/bin/bash
# full GPU test suite + the default bench line (round 2)
mkdir -p gpurun_out
python -c "from paper_conf_asplos_xiazswwyfc24_b200.build import build; build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu_full.txt 2>&1
echo "rc=$?" >> gpurun_out/pytest_gpu_full.txt
timeout 300 python tools/graph_timing.py > gpurun_out/graph_timing.json 2> gpurun_out/graph_timing.err
timeout 1200 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
echo done
