"""The bench's model sequence in one process (BERT, LSTM, MMoE, then Swin-B repeatedly) to catch
interactions between the persistent kernels.  usage: python tools/stress_sequence.py [swin_runs]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402

runs = int(sys.argv[1]) if len(sys.argv) > 1 else 20
which = sys.argv[2] if len(sys.argv) > 2 else "bert,lstm,mmoe"
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
t0 = time.time()
if "bert" in which:
    g, plan, sess, X, y, x = bench.build_bert(0)
    for _ in range(5):
        sess.run()
    torch.cuda.synchronize()
    print("bert ok", round(time.time() - t0, 1), flush=True)
if "lstm" in which:
    lplan, lsess, _ = bench.build_lstm(0)
    for _ in range(3):
        lsess.run()
    torch.cuda.synchronize()
    print("lstm ok", round(time.time() - t0, 1), flush=True)
if "mmoe" in which:
    mplan, msess = bench.build_mmoe(0)
    for _ in range(3):
        msess.run()
    torch.cuda.synchronize()
    print("mmoe ok", round(time.time() - t0, 1), flush=True)
splan, ssess, _ = bench.build_swin(0)
print("swin plan", round(time.time() - t0, 1), flush=True)
for i in range(runs):
    flush.zero_()
    ssess.run()
    torch.cuda.synchronize()
    print("swin run", i, round(time.time() - t0, 2), flush=True)
print("ok")
