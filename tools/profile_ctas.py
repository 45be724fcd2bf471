"""Per-CTA timelines of selected stages (debug marks): which CTAs finish last and why."""
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
n = plan.exec_info()["stages"]
import ctypes as C
cap = 9 * n + 1 + 4 * 160 * n
buf = (C.c_uint64 * cap)()
got = C.c_int32()
L.check(plan.lib.souffle_plan_read_profile_raw(plan.h, C.c_void_p(s.ws.data_ptr()), buf, cap, C.byref(got)))
starts = list(buf[: n + 1])
kinds = [ln.split()[2] if ln.strip().startswith("||") else ln.split()[1]
         for ln in plan.describe().splitlines() if ln.startswith("  ")]
base = 9 * n + 1
for st in range(min(n, 8)):
    t0 = starts[st]
    rows = []
    for c in range(148):
        m = [buf[base + (st * 160 + c) * 4 + k] for k in range(4)]
        rel = [((v - t0) / 1e3 if v >= t0 and v > 0 else None) for v in m]
        if rel[3] is not None:
            rows.append((rel[3], c, rel))
    rows.sort()
    if not rows:
        continue
    print(f"stage {st} {kinds[st]}: n={len(rows)} done min {rows[0][0]:.2f} median {rows[len(rows)//2][0]:.2f} max {rows[-1][0]:.2f}")
    for r in rows[-4:]:
        print("   cta", r[1], " ".join("-" if v is None else f"{v:.2f}" for v in r[2]))
