"""SM clock during the persistent kernel: clock64 vs %globaltimer at every stage start (CTA 0)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L, models as M
from paper_conf_asplos_xiazswwyfc24_b200.session import session
reps = int(sys.argv[1]) if len(sys.argv) > 1 else 3
cfg = dict(synth.BERT_BASE)
x, w = synth.bert_input(cfg), synth.bert_weights(cfg)
g, X, plist, y = M.bert(cfg)
feed = {X: x}
for names, wl in zip(plist, w):
    for k, t in names.items():
        feed[t] = wl[k]
plan = g.partition(L.device_query(0))
plan.set_profiling(True)
s = session(g, plan, feed, [y])
for _ in range(reps):
    s.run()
torch.cuda.synchronize()
starts, marks = plan.read_profile_raw(s.ws.data_ptr())
n = len(marks)
for i in (0, 1, 10, 40, 80):
    if i + 1 < n:
        dt = starts[i + 1] - starts[i]
        dc = marks[i + 1][6] - marks[i][6]
        print(f"stage {i}: {dt / 1e3:.2f} us, {dc} cycles -> {dc / dt:.3f} GHz")
tot_t = starts[n - 1] - starts[0]; tot_c = marks[n - 1][6] - marks[0][6]
print(f"whole run: {tot_t / 1e3:.1f} us at {tot_c / tot_t:.3f} GHz (reps={reps})")
