timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/b7.log 2>&1; echo rc=$? >> gpurun_out/b7.log
