"""Per-step timeline of one CTA of the persistent LSTM kernel (debug stamps, %globaltimer).

usage: SOUFFLE_LSTM_PROF_CTA=<cta> python tools/profile_lstm.py"""
import ctypes as C
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import models as M  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402

cfg = synth.LSTM_CFG
x = synth.lstm_input(cfg)
ps = synth.lstm_params(cfg)
g, nm, top, hs, cs = M.lstm(cfg)
feed = {nm["X"]: x}
for n, p in enumerate(ps):
    feed[nm[f"W{n}"]], feed[nm[f"U{n}"]] = p["W"], p["U"]
    feed[nm[f"bih{n}"]], feed[nm[f"bhh{n}"]] = p["b_ih"], p["b_hh"]
    feed[nm[f"h0_{n}"]] = np.zeros((1, cfg["hidden"]), np.float32)
    feed[nm[f"c0_{n}"]] = np.zeros((1, cfg["hidden"]), np.float32)
plan = g.partition(L.device_query(0))
plan.set_profiling(True)
s = session(g, plan, feed, list(top) + list(hs) + list(cs))
for _ in range(3):
    s.run()
torch.cuda.synchronize()
T = cfg["steps"]
buf = (C.c_uint64 * (4 * T))()
got = C.c_int32()
L.check(plan.lib.souffle_plan_read_profile_raw(plan.h, C.c_void_p(s.ws.data_ptr()), buf, 4 * T, C.byref(got)))
st = np.array(list(buf), dtype=np.float64).reshape(T, 4) / 1.965   # SM cycles -> ns (1965 MHz under load)
t0 = st[0, 0]
for t in list(range(0, 6)) + list(range(T - 3, T)):
    print(f"t={t:3d} start {(st[t,0]-t0)/1e3:8.2f} operands +{(st[t,1]-st[t,0])/1e3:5.2f} gemv +{(st[t,2]-st[t,1])/1e3:5.2f}"
          f" cell+publish +{(st[t,3]-st[t,2])/1e3:5.2f} next-start +{((st[t+1,0]-st[t,3])/1e3 if t + 1 < T else 0):5.2f}")
d = np.diff(st[:, 0]) / 1e3
print("mean step", d.mean(), "operands wait mean", ((st[:, 1] - st[:, 0]) / 1e3).mean(), "gemv mean",
      ((st[:, 2] - st[:, 1]) / 1e3).mean(), "cell+publish mean", ((st[:, 3] - st[:, 2]) / 1e3).mean())
