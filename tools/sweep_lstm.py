"""LSTM latency for several CTAs-per-layer counts (SOUFFLE_LSTM_NP), median of 20 L2-flushed runs.
usage: python tools/sweep_lstm.py 8 12 14"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import sys, statistics, torch
sys.path.insert(0, %r)
import bench
plan, sess, cfg = bench.build_lstm(0)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
t = bench.time_steps(sess, 20, 3, flush, torch.cuda.current_stream())
print("RESULT", statistics.median(t) * 1e3, plan.describe().splitlines()[1][:140])
'''
for np_ in sys.argv[1:]:
    env = dict(os.environ)
    if np_ != "auto":
        env["SOUFFLE_LSTM_NP"] = np_
    out = subprocess.run([sys.executable, "-c", CHILD % ROOT], env=env, capture_output=True, text=True, timeout=300)
    line = [l for l in out.stdout.splitlines() if l.startswith("RESULT")]
    print(np_, line[0] if line else out.stderr[-600:], flush=True)
