"""PAPER.md Fig. 6 on B200: the EfficientNet squeeze-and-excitation sub-modules M0-M9 through the same
C ABI in the paper's four versions -- (a) unfused: one launch per TE (V0); (b) fused: the generic
fused subprograms, one launch per stage (NO_GLOBAL_SYNC); (c) global sync: one persistent launch
(the pattern kernel re-reading x from global); (d) data reuse: the same with x kept in shared
memory -- plus the generic executor's one-launch global-sync lowering.  Median of 30 L2-flushed runs.
Prints one JSON object per module; usage: python tools/ablation_se.py [out.jsonl]"""
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

VERSIONS = [("unfused", L.FLAG_UNFUSED), ("fused", L.FLAG_NO_PATTERN | L.FLAG_NO_GLOBAL_SYNC),
            ("generic_global_sync", L.FLAG_NO_PATTERN), ("global_sync", L.FLAG_NO_PREFETCH), ("data_reuse", 0)]


def run(out_path=None):
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    st = torch.cuda.current_stream()
    rows = []
    for cfg in synth.SE_CONFIGS:
        x, p = synth.se_input(cfg), synth.se_params(cfg)
        g, names, gx, gy = M.se_module(cfg)
        row = {"module": cfg["name"], "hw": cfg["hw"], "channels": cfg["channels"], "squeeze": cfg["squeeze"]}
        for name, flags in VERSIONS:
            plan = g.partition(L.device_query(0), flags)
            s = session(g, plan, {names[k]: p[k] for k in p} | {gx: x}, [gy])
            ts = bench.time_steps(s, 30, 5, flush, st)
            row[name + "_us"] = statistics.median(ts) * 1e3
            row[name + "_launches"] = plan.exec_info()["launches"]
            del s, plan
        row["speedup_data_reuse_vs_unfused"] = row["unfused_us"] / row["data_reuse_us"]
        row["speedup_global_sync_vs_unfused"] = row["unfused_us"] / row["global_sync_us"]
        rows.append(row)
        print(json.dumps(row), flush=True)
    if out_path:
        with open(out_path, "w") as f:
            for r in rows:
                f.write(json.dumps(r) + "\n")
    return rows


if __name__ == "__main__":
    run(sys.argv[1] if len(sys.argv) > 1 else None)
