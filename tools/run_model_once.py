"""Run one model a few times through the C ABI (target for ncu captures).
usage: python tools/run_model_once.py bert|lstm|mmoe|swin [runs]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402

which = sys.argv[1]
runs = int(sys.argv[2]) if len(sys.argv) > 2 else 3
if which == "bert":
    sess = bench.build_bert(0)[2]
elif which == "lstm":
    sess = bench.build_lstm(0)[1]
elif which == "mmoe":
    sess = bench.build_mmoe(0)[1]
else:
    sess = bench.build_swin(0)[1]
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for _ in range(runs):
    flush.zero_()
    sess.run()
torch.cuda.synchronize()
print("ok", which)
