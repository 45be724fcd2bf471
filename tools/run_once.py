"""Run BERT (or a given config) through the fused path a few times (for ncu captures)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L, models as M
from paper_conf_asplos_xiazswwyfc24_b200.session import session
which = sys.argv[1] if len(sys.argv) > 1 else "bert_base"
flags = int(sys.argv[2]) if len(sys.argv) > 2 else 0
layers = int(sys.argv[3]) if len(sys.argv) > 3 else None
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 2
cfg = synth.BERT_BASE if which == "bert_base" else synth.BERT_TINY
if layers:
    cfg = dict(cfg, layers=layers)
x, w = synth.bert_input(cfg), synth.bert_weights(cfg)
g, X, plist, y = M.bert(cfg)
feed = {X: x}
for names, wl in zip(plist, w):
    for k, t in names.items():
        feed[t] = wl[k]
plan = g.partition(L.device_query(0), flags)
s = session(g, plan, feed, [y])
for _ in range(reps):
    s.run()
torch.cuda.synchronize()
print("done")
