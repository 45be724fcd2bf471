"""Per-stage time of Swin-B (batch 1) on the generic fused-subprogram executor, aggregated by stage kind
(globaltimer marks of CTA 0; the describe() text names each stage).  usage: python tools/profile_swin.py"""
import collections
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth.swin as S  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import models as M  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402

cfg = dict(S.SWIN_B, batch=int(sys.argv[1]) if len(sys.argv) > 1 else 1)
fv = S.swin_feed_values(cfg, S.swin_params(cfg))
g, names, x, y = M.swin(cfg)
feed = {names[k]: v for k, v in fv.items()}
feed[x] = S.swin_input(cfg)
plan = g.partition(L.device_query(0))
plan.set_profiling(True)
s = session(g, plan, feed, [y])
for _ in range(3):
    s.run()
torch.cuda.synchronize()
durs = plan.read_profile(s.ws.data_ptr())
lines = [ln for ln in plan.describe().splitlines() if ln.startswith("  ")]
agg = collections.defaultdict(float)
cnt = collections.Counter()
rows = []
for i, ln in enumerate(lines[:len(durs)]):
    parts = ln.split()
    kind = parts[2] if parts[0] == "||" else parts[1]
    agg[kind] += durs[i]
    cnt[kind] += 1
    rows.append((durs[i], i, ln.strip()[:150]))
print("total us", sum(durs), "stages", len(durs))
for k in sorted(agg, key=lambda k: -agg[k]):
    print(f"{k:10s} n={cnt[k]:4d} total {agg[k]:9.1f} us")
print("slowest stages:")
for d, i, ln in sorted(rows, reverse=True)[:25]:
    print(f"{d:8.1f} us  {ln}")
