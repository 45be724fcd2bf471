"""Summarise an ncu report (--set full) and a launch list into profiles/ (run here, no GPU).

usage: python tools/ncu_summary.py <report.ncu-rep> <launches.csv|-> <out-prefix> [kernel-regex]
Writes <out-prefix>.json (key metrics per profiled kernel, dram bytes per launch) and
<out-prefix>_launches.csv (kernel name, device time ns) and prints a short text summary."""
import csv
import io
import json
import re
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__inst_executed.sum", "sm__cycles_elapsed.avg.per_second"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "usecond": 1e-6, "ms": 1e-3,
         "msecond": 1e-3, "nsecond": 1e-9, "s": 1}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                d[k] = v * SCALE.get(units[i], 1) if units[i] in SCALE else v
                d[k + ".unit"] = "s" if units[i] in ("ns", "us", "ms", "usecond", "msecond", "nsecond") else (
                    "byte" if "byte" in units[i] else units[i])
        if "dram__bytes_read.sum" in d:
            d["dram_bytes_per_launch"] = d["dram__bytes_read.sum"] + d.get("dram__bytes_write.sum", 0)
        res.append(d)
    return res


def launches(path):
    rows = list(csv.reader(open(path)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    out = []
    for r in rows[start + 1:]:
        if len(r) < len(hdr) or r[hdr.index("Metric Name")] != "gpu__time_duration.sum":
            continue
        v = float(r[hdr.index("Metric Value")].replace(",", ""))
        unit = r[hdr.index("Metric Unit")]
        out.append((r[hdr.index("Kernel Name")], v * {"ns": 1, "us": 1e3, "ms": 1e6}.get(unit, 1)))
    return out


def main():
    rep, lc, prefix = sys.argv[1:4]
    pat = re.compile(sys.argv[4]) if len(sys.argv) > 4 else None
    summ = {"report": rep.split("/")[-1], "kernels": raw(rep)}
    if lc != "-":
        ls = launches(lc)
        with open(prefix + "_launches.csv", "w") as f:
            w = csv.writer(f)
            w.writerow(["kernel", "ns"])
            for k, v in ls:
                w.writerow([k, v])
        tot = sum(v for _, v in ls)
        mine = [(k, v) for k, v in ls if pat is None or pat.search(k)]
        summ["launch_list"] = {"launches": len(ls), "total_ns": tot, "ours": len(mine),
                               "ours_ns": sum(v for _, v in mine),
                               "ours_share": (sum(v for _, v in mine) / tot) if tot else None}
    if summ["kernels"]:
        summ["dram_bytes_per_launch"] = summ["kernels"][0].get("dram_bytes_per_launch")
    json.dump(summ, open(prefix + ".json", "w"), indent=1)
    print(json.dumps(summ, indent=1)[:3000])


if __name__ == "__main__":
    main()
