"""Per-stage device timeline of the persistent kernel (debug: souffle_plan_set_profiling).

usage: python tools/profile_stages.py [bert_base|bert_tiny|lstm|mmoe] [flags] [layers]
Prints one line per stage (kind, duration us incl. the following grid barrier) and totals per kind."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import models as M  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402


def bert_feed(X, plist, x, w):
    f = {X: x}
    for names, wl in zip(plist, w):
        for k, t in names.items():
            f[t] = wl[k]
    return f


def main():
    which = sys.argv[1] if len(sys.argv) > 1 else "bert_base"
    flags = int(sys.argv[2]) if len(sys.argv) > 2 else 0
    layers = int(sys.argv[3]) if len(sys.argv) > 3 else None
    cfg = synth.BERT_BASE if which == "bert_base" else synth.BERT_TINY
    if layers:
        cfg = dict(cfg, layers=layers)
    x, w = synth.bert_input(cfg), synth.bert_weights(cfg)
    g, X, plist, y = M.bert(cfg)
    plan = g.partition(L.device_query(0), flags)
    plan.set_profiling(True)
    s = session(g, plan, bert_feed(X, plist, x, w), [y])
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(3):
        flush.zero_()
        s.run()
    torch.cuda.synchronize()
    prof = plan.read_profile(s.ws.data_ptr())
    txt = plan.describe()
    if txt.startswith("pattern bert:") and "not used" not in txt.splitlines()[0]:
        kinds = ["CVT"] + ["QKV", "ATTNO", "LN1", "FFN1", "FFN2", "LN2"] * cfg["layers"]
    else:
        kinds = [ln.split()[2] if ln.strip().startswith("||") else ln.split()[1]
                 for ln in txt.splitlines() if ln.startswith("  ")]
    tot = {}
    for i, (k, t) in enumerate(zip(kinds, prof)):
        tot[k] = tot.get(k, 0.0) + t
        if i < 16:
            print(f"{i:3d} {k:10s} {t:9.2f} us")
    print("total", sum(prof), "us;", {k: round(v, 1) for k, v in tot.items()})


if __name__ == "__main__":
    main()
