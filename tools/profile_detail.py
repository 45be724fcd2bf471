"""Intra-stage timeline of CTA 0 for the first layer of BERT-base (debug marks, ns -> us)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L, models as M
from paper_conf_asplos_xiazswwyfc24_b200.session import session
layers = int(sys.argv[1]) if len(sys.argv) > 1 else 2
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
    flush.zero_(); s.run()
torch.cuda.synchronize()
starts, marks = plan.read_profile_raw(s.ws.data_ptr())
kinds = [ln.split()[2] if ln.strip().startswith("||") else ln.split()[1]
         for ln in plan.describe().splitlines() if ln.startswith("  ")]
t0 = starts[0]
for i in range(min(len(kinds), 16)):
    st = (starts[i] - t0) / 1e3
    dur = (starts[i + 1] - starts[i]) / 1e3
    mk = " ".join(f"m{k}={(m - starts[i]) / 1e3:7.2f}" for k, m in enumerate(marks[i]) if m >= starts[i] and m > 0)
    print(f"{i:3d} {kinds[i]:9s} start {st:8.2f} dur {dur:7.2f} | {mk}")
