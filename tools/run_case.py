"""Debug helper: run one model config through the fused path and compare with the oracle."""
import sys
import numpy as np
import synth
from oracle import graphs as og, te
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L, models as M
from paper_conf_asplos_xiazswwyfc24_b200.session import session

which = sys.argv[1]
flags = int(sys.argv[2]) if len(sys.argv) > 2 else 0
if which.startswith("bert"):
    cfg = synth.BERT_TINY if which == "bert_tiny" else dict(synth.BERT_BASE, layers=int(sys.argv[3]) if len(sys.argv) > 3 else 1)
    x = synth.bert_input(cfg); w = synth.bert_weights(cfg)
    spec, X, plist, y = og.bert(cfg)
    ref = te.evaluate(spec, og.bert_feed(X, plist, x, w), bf16_operands=cfg["gemm_dtype"] == "bf16")[y]
    g, gX, gpl, gy = M.bert(cfg)
    plan = g.partition(L.device_query(0), flags)
    print(plan.describe())
    s = session(g, plan, og.bert_feed(gX, gpl, x, w), [gy])
    s.run()
    out = s.result(gy)
    print("max abs err", np.abs(out - ref).max(), "ref max", np.abs(ref).max())
