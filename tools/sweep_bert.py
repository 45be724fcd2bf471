"""Tile-policy sweep of the BERT kernel (env overrides SOUFFLE_BERT_QKV / FFN1 / FFN2), median latency of
20 L2-flushed runs.  usage: python tools/sweep_bert.py "QKV=16,FFN1=32" "QKV=32" ..."""
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CHILD = r'''
import os, sys, statistics, torch
sys.path.insert(0, %r)
import bench
g, plan, sess, X, y, x = bench.build_bert(0)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
t = bench.time_steps(sess, 30, 5, flush, torch.cuda.current_stream())
print("RESULT", statistics.median(t) * 1e3, plan.describe().splitlines()[2:6])
'''
for spec in sys.argv[1:]:
    env = dict(os.environ)
    for kv in spec.split(";"):
        if kv:
            k, v = kv.split("=", 1)
            env["SOUFFLE_BERT_" + k] = v
    out = subprocess.run([sys.executable, "-c", CHILD % ROOT], env=env, capture_output=True, text=True, timeout=300)
    line = [l for l in out.stdout.splitlines() if l.startswith("RESULT")]
    print(spec, line[0] if line else out.stderr[-500:], flush=True)
