"""Phase timeline of the MBConv pattern kernel (CTA 0, %globaltimer; SOUFFLE_MB_PROF=1 is set here).
usage: python tools/profile_mbconv.py [module indices...]"""
import os
import sys

os.environ["SOUFFLE_MB_PROF"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import models as M  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402

names = ["expand", "sync0", "depthwise+pool", "sync1", "SE (pooled, fc1, gates start)", "project (+ split-K finish)"]
for i in [int(a) for a in sys.argv[1:]] or range(10):
    cfg = synth.MBCONV_CONFIGS[i]
    g, nm, gx, gy = M.mbconv(cfg)
    plan = g.partition(L.device_query(0))
    p = {**synth.mbconv_params(cfg), **synth.mbconv_masks(cfg)}
    s = session(g, plan, {nm[k]: v for k, v in p.items()} | {gx: synth.mbconv_input(cfg)}, [gy])
    rows = []
    for _ in range(5):
        s.run()
        torch.cuda.synchronize()
        rows.append(s.ws[64:128].view(torch.int64).cpu().numpy().astype(np.float64))
    t = np.median(np.stack(rows), 0)
    t1 = t[1] if cfg["expand"] != 1 else t[0]
    seg = [t1 - t[0], t[2] - t1, t[3] - t[2], t[4] - t[3], t[5] - t[4], t[6] - t[5]]
    print(cfg["name"], "total %.1f us |" % ((t[6] - t[0]) / 1e3),
          " ".join(f"{n} {v / 1e3:.1f}" for n, v in zip(names, seg)))
