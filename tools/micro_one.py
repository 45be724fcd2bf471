import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L
from paper_conf_asplos_xiazswwyfc24_b200.session import session
rows, cols, n, flags = (int(a) for a in sys.argv[1:5])
g = L.Graph(); x = g.placeholder((rows, cols), L.F32, const=False); h = x
for _ in range(n): h = g.ew("neg", h)
g.mark_output(h)
plan = g.partition(L.device_query(0), flags)
s = session(g, plan, {x: np.ones((rows, cols), np.float32)}, [h])
for _ in range(3): s.run()
torch.cuda.synchronize(); print("ok")
