"""PAPER.md Fig. 5 / 6 on B200 with the whole MBConv block as the sub-module (tests/test_oracle_mbconv.py
pins the TE program to torchvision): M0-M9 in (a) unfused: one launch per TE; (b) fused: the generic
executor's fused stages launched one by one (NO_GLOBAL_SYNC); the generic executor with one launch per
subprogram, without and with §6.5 reuse; (c) global sync: the MBConv pattern kernel, one persistent
launch (kernels/mbconv.cu, NO_PREFETCH: d through L2); (d) data reuse: the same kernel with each CTA's
d block kept in shared memory (where the planner chooses it).
Median of 30 L2-flushed runs; one JSON object per module.  usage: python tools/ablation_mbconv.py [out.jsonl]"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import _lib as L  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200 import models as M  # noqa: E402
from paper_conf_asplos_xiazswwyfc24_b200.session import session  # noqa: E402

VERSIONS = [("unfused", L.FLAG_UNFUSED), ("fused", L.FLAG_NO_GLOBAL_SYNC),
            ("generic_global_sync", L.FLAG_NO_PATTERN | L.FLAG_NO_PREFETCH), ("generic_reuse", L.FLAG_NO_PATTERN),
            ("global_sync", L.FLAG_NO_PREFETCH), ("data_reuse", 0)]


def run(out_path=None):
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    st = torch.cuda.current_stream()
    rows = []
    for cfg in synth.MBCONV_CONFIGS:
        p = {**synth.mbconv_params(cfg), **synth.mbconv_masks(cfg)}
        g, names, gx, gy = M.mbconv(cfg)
        row = {k: cfg[k] for k in ("name", "cin", "cout", "expand", "k", "stride", "hw")}
        for name, flags in VERSIONS:
            plan = g.partition(L.device_query(0), flags)
            s = session(g, plan, {names[k]: v for k, v in p.items()} | {gx: synth.mbconv_input(cfg)}, [gy])
            ts = bench.time_steps(s, 30, 5, flush, st)
            info = plan.exec_info()
            row[name + "_us"] = statistics.median(ts) * 1e3
            row[name + "_launches"] = info["launches"]
            row[name + "_barriers"] = info["barriers"]
            del s, plan
        for name in ("fused", "generic_global_sync", "generic_reuse", "global_sync", "data_reuse"):
            row["speedup_" + name + "_vs_unfused"] = row["unfused_us"] / row[name + "_us"]
        rows.append(row)
        print(json.dumps(row), flush=True)
    if out_path:
        with open(out_path, "w") as f:
            for r in rows:
                f.write(json.dumps(r) + "\n")
    return rows


if __name__ == "__main__":
    run(sys.argv[1] if len(sys.argv) > 1 else None)
