"""In-graph timeline of the Swin pattern launches (SOUFFLE_SWIN_TRACE: every launch stamps
%globaltimer at its start); prints per-launch-kind totals.  usage: python tools/swin_trace.py [batch]"""
import collections
import os
import sys

os.environ["SOUFFLE_SWIN_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402

batch = int(sys.argv[1]) if len(sys.argv) > 1 else 1
plan, sess, cfg = bench.build_swin(0, batch=batch)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for _ in range(5):
    flush.zero_()
    sess.run()
torch.cuda.synchronize()
off, nb = plan.debug_region("trace")
t = sess.ws[off:off + nb].view(torch.int64).cpu().numpy().astype(np.float64)
d = np.diff(t) / 1e3
kinds = ["bias", "im2col", "gemm_pe", "ln_pe"]
for s, depth in enumerate(cfg["depths"]):
    kinds += ["ln1", "qkv", "attn", "proj", "ln2", "fc1", "fc2"] * depth
    if s + 1 < len(cfg["depths"]):
        kinds += ["ln_merge", "gemm_merge"]
kinds += ["pool", "head"]
tot = collections.defaultdict(float)
for k, v in zip(kinds, d):
    tot[k] += v
print(f"batch {batch}: first launch -> last launch start {(t[-1] - t[0]) / 1e3:.1f} us over {len(t)} launches")
for k in sorted(tot, key=lambda k: -tot[k]):
    print(f"  {k:10s} {tot[k]:8.1f} us")
per = [f"{k}:{v:.1f}" for k, v in zip(kinds, d)]
print("stage-3 block 0:", per[4 + 14 + 2 + 14 + 2: 4 + 14 + 2 + 14 + 2 + 7])
