"""Sub-stage marks (CTA 0) of the first Swin-B stages on the generic executor.
usage: python tools/profile_swin_marks.py [nstages]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth.swin as S  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import models as M  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402

cfg = S.SWIN_B
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
starts, marks = plan.read_profile_raw(s.ws.data_ptr())
lines = [ln for ln in plan.describe().splitlines() if ln.startswith("  ")]
n = int(sys.argv[1]) if len(sys.argv) > 1 else 24
for i in range(min(n, len(lines))):
    dur = (starts[i + 1] - starts[i]) / 1e3
    mk = " ".join(f"m{k}={(m - starts[i]) / 1e3:6.2f}" for k, m in enumerate(marks[i]) if m >= starts[i] and m > 0)
    print(f"{dur:7.2f} us | {mk} | {lines[i].strip()[:110]}")
