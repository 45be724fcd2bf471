"""One small launch of a kernel family, checked against the oracle (for compute-sanitizer runs).
usage: python tools/san_case.py bert_small | swin_small | generic_tiny | rowwise | swin_generic | mbconv:IDX |
       lstm_small | mmoe
(rowwise / swin_generic / generic_tiny exercise the generic executor's row-block stages and tensor cache;
SOUFFLE_CACHE_FLOATS=2048 forces LRU spills)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import synth  # noqa: E402
import synth.swin as SW  # noqa: E402
from oracle import graphs as og  # noqa: E402
from oracle import te  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import models as M  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402

which = sys.argv[1]
if which in ("bert_small", "generic_tiny"):
    cfg = dict(synth.BERT_BASE, seq=32, hidden=256, heads=4, ffn=1024, layers=2) if which == "bert_small" else synth.BERT_TINY
    x, w = synth.bert_input(cfg), synth.bert_weights(cfg)
    spec, X, plist, y = og.bert(cfg)
    ref = te.evaluate(spec, og.bert_feed(X, plist, x, w), bf16_operands=cfg["gemm_dtype"] == "bf16")[y]
    g, gX, gpl, gy = M.bert(cfg)
    plan = g.partition(L.device_query(0))
    s = session(g, plan, og.bert_feed(gX, gpl, x, w), [gy])
    s.run()
    out = s.result(gy)
elif which.startswith("mbconv:"):
    cfg = synth.MBCONV_CONFIGS[int(which.split(":")[1])]
    p = {**synth.mbconv_params(cfg), **synth.mbconv_masks(cfg)}
    spec, on, ox, oy = og.mbconv(cfg)
    x = synth.mbconv_input(cfg)
    ref = te.evaluate(spec, {on[k]: v for k, v in p.items()} | {ox: x})[oy]
    g, gn, gx, gy = M.mbconv(cfg)
    plan = g.partition(L.device_query(0))
    s = session(g, plan, {gn[k]: v for k, v in p.items()} | {gx: x}, [gy])
    s.run()
    s.run()
    out = s.result(gy)
elif which in ("lstm_small", "mmoe"):
    if which == "lstm_small":   # register-resident GEMV kernel (3 layers x 64 units x 5 steps)
        cfg = dict(synth.LSTM_CFG, steps=5, layers=3, hidden=64, input=64, w_dtype="f32")
        x, ps = synth.lstm_input(cfg), synth.lstm_params(cfg)
        spec, names, top, hs, cs = og.lstm(cfg)

        def feed_for(nm):
            f = {nm["X"]: x}
            for n, q in enumerate(ps):
                f[nm[f"W{n}"]], f[nm[f"U{n}"]] = q["W"], q["U"]
                f[nm[f"bih{n}"]], f[nm[f"bhh{n}"]] = q["b_ih"], q["b_hh"]
                f[nm[f"h0_{n}"]] = np.zeros((1, cfg["hidden"]), np.float32)
                f[nm[f"c0_{n}"]] = np.zeros((1, cfg["hidden"]), np.float32)
            return f
        ref = te.evaluate(spec, feed_for(names))[top[-1]]
        g, gn, gtop, ghs, gcs = M.lstm(cfg)
        plan = g.partition(L.device_query(0))
        s = session(g, plan, feed_for(gn), [gtop[-1]])
        s.run()
        s.run()
        out = s.result(gtop[-1])
    else:                       # 8-CTA cluster kernel
        cfg = synth.MMOE_CFG
        p, x = synth.mmoe_params(cfg), synth.mmoe_input(cfg)
        spec, names, outs = og.mmoe(cfg)
        feed = {names[k]: v for k, v in p.items()}
        feed[names["x"]] = x
        ref = te.evaluate(spec, feed)[outs[0]]
        g, gn, gouts = M.mmoe(cfg)
        gfeed = {gn[k]: v for k, v in p.items()}
        gfeed[gn["x"]] = x
        plan = g.partition(L.device_query(0))
        s = session(g, plan, gfeed, gouts)
        s.run()
        out = s.result(gouts[0])
    print(plan.describe().splitlines()[1 if which == "lstm_small" else 2][:160])
elif which == "rowwise":
    spec = synth.random_rowwise_spec(0)
    ins = synth.spec_inputs(spec, 0)
    g = M.from_spec(spec)
    plan = g.partition(L.device_query(0))
    s = session(g, plan, ins, spec["outputs"])
    s.run()
    o = spec["outputs"][0]
    out, ref = s.result(o), te.evaluate(spec, ins)[o]
else:
    cfg = dict(SW.SWIN_TINY, embed=128, heads=(4, 8), gemm_dtype="bf16") if which == "swin_small" else \
        dict(SW.SWIN_TINY, batch=1)
    P = SW.swin_params(cfg)
    fv = SW.swin_feed_values(cfg, P)
    img = SW.swin_input(cfg)
    g, names, gx, gy = M.swin(cfg)
    feed = {names[k]: v for k, v in fv.items()}
    feed[gx] = img
    plan = g.partition(L.device_query(0))
    s = session(g, plan, feed, [gy])
    s.run()
    out = s.result(gy)
    spec, on, ox, oy = og.swin(cfg)
    ref = te.evaluate(spec, feed, bf16_operands=cfg.get("gemm_dtype") == "bf16")[oy]
info = [ln for ln in plan.describe().splitlines() if ln.startswith(("plan:", "tensor cache"))]
print(which, info, "max abs err", float(np.abs(out - ref).max()))
