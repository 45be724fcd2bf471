import sys, numpy as np
sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
import synth
from oracle import graphs as og, te
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L, models as M
from paper_conf_asplos_xiazswwyfc24_b200.session import session
import torch
steps, layers, hidden = [int(a) for a in sys.argv[1:4]]
cfg = dict(synth.LSTM_CFG, steps=steps, layers=layers, hidden=hidden, input=hidden, w_dtype="f32")
g, nm, top, hs, cs = M.lstm(cfg)
feed = {nm["X"]: synth.lstm_input(cfg)}
for n, p in enumerate(synth.lstm_params(cfg)):
    feed[nm[f"W{n}"]], feed[nm[f"U{n}"]] = p["W"], p["U"]
    feed[nm[f"bih{n}"]], feed[nm[f"bhh{n}"]] = p["b_ih"], p["b_hh"]
    feed[nm[f"h0_{n}"]] = np.zeros((1, cfg["hidden"]), np.float32)
    feed[nm[f"c0_{n}"]] = np.zeros((1, cfg["hidden"]), np.float32)
for flags in [L.FLAG_NO_PATTERN, L.FLAG_NO_GLOBAL_SYNC | L.FLAG_NO_PATTERN]:
    plan = g.partition(L.device_query(0), flags)
    print(flags, plan.exec_info(), flush=True)
    s = session(g, plan, feed, list(top))
    s.run()
    torch.cuda.synchronize()
    print("ok", flags, s.result(top[-1])[0, :4], flush=True)
