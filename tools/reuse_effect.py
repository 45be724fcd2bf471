"""Measured effect of §6.5 tensor reuse on the generic executor: the same TE
program planned with reuse (row-block affinity: CTA-local dependencies without grid barriers, LRU
shared-memory tensor cache) and without it (SOUFFLE_FLAG_NO_PREFETCH), median of L2-flushed runs.
usage: python tools/reuse_effect.py [swin bert swin_tiny rowwise]  -> JSON lines on stdout"""
import json
import os
import re
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import synth  # noqa: E402
import synth.swin as SW  # noqa: E402
from ablation import graph_and_feed, time_plan  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import models as M  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402


def workloads(names):
    for name in names:
        if name in ("swin", "bert"):
            g, feed, outs = graph_and_feed(name)
            yield name + " (generic V3)", g, feed, outs, L.FLAG_NO_PATTERN
        elif name == "swin_tiny":
            cfg = dict(SW.SWIN_TINY, batch=1)
            fv = SW.swin_feed_values(cfg, SW.swin_params(cfg))
            g, nm, x, y = M.swin(cfg)
            feed = {nm[k]: v for k, v in fv.items()}
            feed[x] = SW.swin_input(cfg)
            yield "swin_tiny fp32", g, feed, [y], 0
        elif name == "rowwise":
            for seed in range(4):
                spec = synth.random_rowwise_spec(seed)
                yield f"rowwise seed {seed}", M.from_spec(spec), synth.spec_inputs(spec, seed), spec["outputs"], 0


def stats(d):
    b = int(re.search(r"(\d+) grid barrier", d).group(1))
    m = re.search(r"tensor cache: (\d+) tensor.*?(\d+) hit.*?(\d+) LRU.*?(\d+) global", d)
    return b, ([int(x) for x in m.groups()] if m else [0, 0, 0, 0])


def main():
    names = sys.argv[1:] or ["swin", "bert", "swin_tiny", "rowwise"]
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for label, g, feed, outs, base in workloads(names):
        row = {"workload": label}
        variants = [("reuse", base, None), ("no_reuse", base | L.FLAG_NO_PREFETCH, None)]
        if os.environ.get("REUSE_SWEEP"):
            variants += [("reuse_cache0", base, "0"), ("reuse_cache88k", base, "22528")]
        for tag, flags, cap in variants:
            if cap is None:
                os.environ.pop("SOUFFLE_CACHE_FLOATS", None)
            else:
                os.environ["SOUFFLE_CACHE_FLOATS"] = cap
            plan = g.partition(L.device_query(0), flags)
            os.environ.pop("SOUFFLE_CACHE_FLOATS", None)
            sess = session(g, plan, feed, outs)
            us = time_plan(sess, 20, flush)
            b, c = stats(plan.describe())
            row[tag] = {"latency_us": round(us, 1), "grid_barriers": b, "cached_tensors": c[0], "hits": c[1],
                        "spills": c[2], "stores_elided": c[3]}
            del sess, plan
            torch.cuda.empty_cache()
        row["speedup"] = round(row["no_reuse"]["latency_us"] / row["reuse"]["latency_us"], 3)
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
