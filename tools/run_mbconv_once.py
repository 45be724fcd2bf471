"""Run one EfficientNet MBConv block through the pattern kernel (for ncu captures).
usage: python tools/run_mbconv_once.py <module index> [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import models as M  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402

cfg = synth.MBCONV_CONFIGS[int(sys.argv[1])]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
g, nm, gx, gy = M.mbconv(cfg)
plan = g.partition(L.device_query(0))
p = {**synth.mbconv_params(cfg), **synth.mbconv_masks(cfg)}
s = session(g, plan, {nm[k]: v for k, v in p.items()} | {gx: synth.mbconv_input(cfg)}, [gy])
for _ in range(reps):
    s.run()
torch.cuda.synchronize()
print("ok", cfg["name"], plan.exec_info())
