mkdir -p gpurun_out
nvidia-smi > gpurun_out/s_nvsmi.txt 2>&1
timeout 1500 python -m pytest tests -q -m gpu -x > gpurun_out/s_pytest_gpu.txt 2>&1; echo "rc=$?" >> gpurun_out/s_pytest_gpu.txt
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/s_bench.json 2> gpurun_out/s_bench.err
timeout 300 python tools/profile_bert.py 12 > gpurun_out/s_timeline.txt 2>&1
echo done
