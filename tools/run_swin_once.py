"""Run Swin-B through the pattern kernels `reps` times at a given batch (for ncu launch lists).
usage: python tools/run_swin_once.py [batch] [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402

batch = int(sys.argv[1]) if len(sys.argv) > 1 else 1
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
plan, sess, cfg = bench.build_swin(0, batch=batch)
for _ in range(reps):
    sess.run()
torch.cuda.synchronize()
print(plan.describe().splitlines()[3][:200] if False else "ok", plan.exec_info())
