"""Table 4 ablation on B200 (Table 4): latency of each model
under the optimisation ladder, through the same C ABI (median of L2-flushed runs, CUDA events).
  V0  unfused: one kernel per TE                      (SOUFFLE_FLAG_UNFUSED)
  V1  + horizontal transformation                     (NO_VERTICAL | NO_GLOBAL_SYNC | NO_PATTERN)
  V2  + vertical transformation                       (NO_GLOBAL_SYNC | NO_PATTERN)
  V3  + global synchronisation: one launch per SP     (NO_PATTERN | NO_PREFETCH: generic executor)
  V3r + §6.5 tensor reuse in the generic executor     (NO_PATTERN: row-block stages, LRU smem cache)
  V4  + the model's pattern kernel (persistent, cross-stage weight prefetch / on-chip weights)
usage: python tools/ablation.py [models...]   (bert lstm mmoe swin) -> JSON lines on stdout"""
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
import synth.swin as SW  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import models as M  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402

VARIANTS = [("V0", L.FLAG_UNFUSED), ("V1", L.FLAG_NO_VERTICAL | L.FLAG_NO_GLOBAL_SYNC | L.FLAG_NO_PATTERN),
            ("V2", L.FLAG_NO_GLOBAL_SYNC | L.FLAG_NO_PATTERN), ("V3", L.FLAG_NO_PATTERN | L.FLAG_NO_PREFETCH),
            ("V3r", L.FLAG_NO_PATTERN), ("V4", 0)]


def graph_and_feed(name):
    if name == "bert":
        cfg = synth.BERT_BASE
        g, X, plist, y = M.bert(cfg)
        feed = {X: synth.bert_input(cfg)}
        for names, wl in zip(plist, synth.bert_weights(cfg)):
            for k, t in names.items():
                feed[t] = wl[k]
        return g, feed, [y]
    if name == "lstm":
        cfg = synth.LSTM_CFG
        g, nm, top, hs, cs = M.lstm(cfg)
        feed = {nm["X"]: synth.lstm_input(cfg)}
        for n, p in enumerate(synth.lstm_params(cfg)):
            feed[nm[f"W{n}"]], feed[nm[f"U{n}"]] = p["W"], p["U"]
            feed[nm[f"bih{n}"]], feed[nm[f"bhh{n}"]] = p["b_ih"], p["b_hh"]
            feed[nm[f"h0_{n}"]] = np.zeros((1, cfg["hidden"]), np.float32)
            feed[nm[f"c0_{n}"]] = np.zeros((1, cfg["hidden"]), np.float32)
        return g, feed, list(top) + list(hs) + list(cs)
    if name == "mmoe":
        cfg = synth.MMOE_CFG
        g, names, outs = M.mmoe(cfg)
        feed = {names[k]: v for k, v in synth.mmoe_params(cfg).items()}
        feed[names["x"]] = synth.mmoe_input(cfg)
        return g, feed, outs
    cfg = SW.SWIN_B
    fv = SW.swin_feed_values(cfg, SW.swin_params(cfg))
    g, names, x, y = M.swin(cfg)
    feed = {names[k]: v for k, v in fv.items()}
    feed[x] = SW.swin_input(cfg)
    return g, feed, [y]


def time_plan(sess, reps, flush):
    ts = []
    for i in range(reps + 2):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        sess.run()
        b.record()
        b.synchronize()
        if i >= 2:
            ts.append(a.elapsed_time(b) * 1e3)
    return statistics.median(ts)


def main():
    models = sys.argv[1:] or ["mmoe", "bert", "lstm", "swin"]
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for name in models:
        g, feed, outs = graph_and_feed(name)
        for vname, flags in VARIANTS:
            t0 = time.time()
            plan = g.partition(L.device_query(0), flags)
            plan_s = time.time() - t0
            sess = session(g, plan, feed, outs)
            info = plan.exec_info()
            reps = 3 if flags == L.FLAG_UNFUSED and name in ("lstm", "swin") else 10
            us = time_plan(sess, reps, flush)
            pat = [ln for ln in plan.describe().splitlines() if ln.startswith("pattern") and "not used" not in ln]
            kernel = (pat[0][:90] if pat else "generic executor (exec.cu)") if flags == 0 else "generic executor (exec.cu)"
            print(json.dumps({"model": name, "variant": vname, "flags": flags, "latency_us": round(us, 1),
                              "launches": info["launches"], "stages": info["stages"], "plan_s": round(plan_s, 2),
                              "kernel": kernel}), flush=True)
            del sess, plan
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
