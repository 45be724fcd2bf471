"""Phase timeline of the ResNeXt pattern kernel (SOUFFLE_RX_PROF: CTA 0 stamps %globaltimer at the phase
boundaries: 1x1 + projection | grouped 3x3 | 1x1 + shortcut).  usage: python tools/profile_resnext.py"""
import os
import sys

os.environ["SOUFFLE_RX_PROF"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import models as M  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402

for cfg in synth.RESNEXT_CONFIGS:
    p = {**synth.resnext_params(cfg), **synth.resnext_masks(cfg)}
    g, names, gx, gy = M.resnext(cfg)
    plan = g.partition(L.device_query(0))
    s = session(g, plan, {names[k]: v for k, v in p.items()} | {gx: synth.resnext_input(cfg)}, [gy])
    for _ in range(5):
        s.run()
    torch.cuda.synchronize()
    t = s.ws[64:64 + 32].view(torch.int64).cpu().tolist()
    print(cfg["name"], "1x1+proj %.1f | grouped 3x3 (+barrier) %.1f | 1x1+shortcut (+barrier) %.1f us" %
          ((t[1] - t[0]) / 1e3, (t[2] - t[1]) / 1e3, (t[3] - t[2]) / 1e3))
