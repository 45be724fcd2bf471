"""Slowest stages of a model on the generic executor (CTA-0 stage marks).
usage: python tools/profile_generic.py <bert|lstm|mmoe|swin|mbconv:IDX> [flags]"""
import collections
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from ablation import graph_and_feed  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402

name = sys.argv[1]
flags = int(sys.argv[2]) if len(sys.argv) > 2 else L.FLAG_NO_PATTERN
if name.startswith("mbconv:"):
    import synth
    from paper_conf_asplos_xiazswwyfc24_b200 import models as M
    cfg = synth.MBCONV_CONFIGS[int(name.split(":")[1])]
    g, nm, gx, gy = M.mbconv(cfg)
    feed = {nm[k]: v for k, v in {**synth.mbconv_params(cfg), **synth.mbconv_masks(cfg)}.items()}
    feed[gx] = synth.mbconv_input(cfg)
    outs = [gy]
    flags = int(sys.argv[2]) if len(sys.argv) > 2 else 0
else:
    g, feed, outs = graph_and_feed(name)
plan = g.partition(L.device_query(0), flags)
plan.set_profiling(True)
s = session(g, plan, feed, outs)
for _ in range(2):
    s.run()
torch.cuda.synchronize()
starts, marks = plan.read_profile_raw(s.ws.data_ptr())
lines = [ln for ln in plan.describe().splitlines() if ln.startswith("  ")]
agg = collections.defaultdict(float)
rows = []
for i in range(len(lines)):
    d = (starts[i + 1] - starts[i]) / 1e3
    parts = lines[i].split()
    kind = parts[2] if parts[0] == "||" else parts[1]
    agg[kind] += d
    mk = " ".join(f"m{k}={(m - starts[i]) / 1e3:.1f}" for k, m in enumerate(marks[i]) if m >= starts[i] and m > 0)
    rows.append((d, lines[i].strip()[:120], mk))
print("total us", (starts[len(lines)] - starts[0]) / 1e3, dict((k, round(v, 1)) for k, v in agg.items()))
for d, ln, mk in sorted(rows, reverse=True)[:15]:
    print(f"{d:9.1f} us  {ln} | {mk}")
