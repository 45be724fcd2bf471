"""Sub-stage timeline of the specialised BERT kernel (debug marks, CTA 0 / first attention CTA).

usage: python tools/profile_bert.py [layers]   (profiling on; timestamps from %globaltimer)"""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import models as M  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402

layers = int(sys.argv[1]) if len(sys.argv) > 1 else 12
noflush = len(sys.argv) > 2 and sys.argv[2] == "warm"
cfg = dict(synth.BERT_BASE, layers=layers)
x, w = synth.bert_input(cfg), synth.bert_weights(cfg)
g, X, plist, y = M.bert(cfg)
feed = {X: x}
for names, wl in zip(plist, w):
    for k, t in names.items():
        feed[t] = wl[k]
plan = g.partition(L.device_query(0))
plan.set_profiling(True)
s = session(g, plan, feed, [y])
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for _ in range(3):
    if not noflush:
        flush.zero_()
    s.run()
torch.cuda.synchronize()
ns = plan.exec_info()["stages"]
cap = 17 * ns + 2
buf = (C.c_uint64 * cap)()
got = C.c_int32()
L.check(plan.lib.souffle_plan_read_profile_raw(plan.h, C.c_void_p(s.ws.data_ptr()), buf, cap, C.byref(got)))
starts = list(buf[:ns]) + [buf[ns + 1]]
kinds = ["CVT"] + ["QKV", "ATTNO", "LN1", "FFN1", "FFN2", "LN2"] * layers
tot = {}
for i in range(ns):
    dur = (starts[i + 1] - starts[i]) / 1e3
    tot[kinds[i]] = tot.get(kinds[i], 0.0) + dur
    if i < 16:
        mk = []
        for k in range(16):
            m = buf[ns + 2 + 16 * i + k]
            if m >= starts[i] and m > 0:
                mk.append(f"m{k}={(m - starts[i]) / 1e3:.2f}")
        print(f"{i:3d} {kinds[i]:5s} dur {dur:6.2f} | " + " ".join(mk))
print("total", (starts[ns] - starts[0]) / 1e3, "us;", {k: round(v, 1) for k, v in tot.items()})
