timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/p9.log 2>&1; echo rc=$? >> gpurun_out/p9.log
