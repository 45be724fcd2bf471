timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "bert_base" > gpurun_out/p5.log 2>&1; echo rc=$? >> gpurun_out/p5.log
timeout 100 python tools/profile_bert.py 2 > gpurun_out/pb6.log 2>&1
timeout 200 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-v0 > gpurun_out/b5.log 2>&1
