"""Table 4 ladder on B200 for the ResNeXt Bottleneck blocks R0-R7 (Table 2 / Table 4:
ResNeXt V0 29.0 -> V1 5.90 -> V2 4.43 ms for the whole network on A100): (V0) unfused, one launch per
TE; (V2) fused stages launched one by one (NO_GLOBAL_SYNC: horizontal + vertical transformations, no
grid barriers); (V3/V4) the generic executor with one launch per subprogram (grid barriers between
dependent stages) and §6.5 reuse.  The grouped 3x3 convolution is already ONE batched matmul TE per tap
(the horizontal form of the 64 group convolutions).  Median of 20 L2-flushed runs, one JSON object per
block.  usage: python tools/ablation_resnext.py [out.jsonl]"""
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

VERSIONS = [("V0_unfused", L.FLAG_UNFUSED), ("V2_fused_no_global_sync", L.FLAG_NO_GLOBAL_SYNC),
            ("V3_generic_global_sync", L.FLAG_NO_PATTERN | L.FLAG_NO_PREFETCH), ("V4_generic_reuse", L.FLAG_NO_PATTERN),
            ("pattern", 0)]


def run(out_path=None):
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    st = torch.cuda.current_stream()
    rows = []
    for cfg in synth.RESNEXT_CONFIGS:
        p = {**synth.resnext_params(cfg), **synth.resnext_masks(cfg)}
        g, names, gx, gy = M.resnext(cfg)
        row = {k: cfg[k] for k in ("name", "cin", "width", "cout", "hw", "stride", "groups")}
        for name, flags in VERSIONS:
            plan = g.partition(L.device_query(0), flags)
            s = session(g, plan, {names[k]: v for k, v in p.items()} | {gx: synth.resnext_input(cfg)}, [gy])
            ts = bench.time_steps(s, 20, 3, flush, st)
            info = plan.exec_info()
            row[name + "_us"] = statistics.median(ts) * 1e3
            row[name + "_launches"] = info["launches"]
            row[name + "_barriers"] = info["barriers"]
            del s, plan
        for name, _ in VERSIONS[1:]:
            row["speedup_" + name + "_vs_unfused"] = row["V0_unfused_us"] / row[name + "_us"]
        rows.append(row)
        print(json.dumps(row), flush=True)
    if out_path:
        with open(out_path, "w") as f:
            for r in rows:
                f.write(json.dumps(r) + "\n")
    return rows


if __name__ == "__main__":
    run(sys.argv[1] if len(sys.argv) > 1 else None)
