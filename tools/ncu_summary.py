"""Summarise ncu outputs brought back in gpurun_out/ into profiles/.

    python tools/ncu_summary.py --launches gpurun_out/launches.csv --out profiles/r01_launches.md
    python tools/ncu_summary.py --rep gpurun_out/prof_x.ncu-rep --out profiles/r01_x.md [--traffic-key NAME]

Launch lists: per kernel name, launches, total/mean device time and share
(cold-cache, serialised: compare shares, not absolutes).  Full captures: the
metrics that decide the roofline (duration, DRAM bytes, tensor-pipe and SM
throughput, occupancy, registers).  --traffic-key also records
dram_bytes_per_launch in profiles/ncu_traffic.json for bench.py.
"""
import argparse
import csv
import io
import json
import os
import subprocess
from collections import defaultdict

import re

PATTERNS = [r"^gpu__time_duration\.sum$", r"^dram__bytes_(read|write)\.sum$", r"^gpu__dram_throughput\.avg\.pct",
            r"^sm__throughput\.avg\.pct", r"tensor.*pct_of_peak", r"^lts__throughput\.avg\.pct_of_peak_sustained_elapsed$",
            r"^launch__registers_per_thread$", r"^sm__warps_active\.avg\.pct_of_peak_sustained_active$",
            r"^launch__grid_size$", r"^launch__block_size$", r"^smsp__inst_executed\.sum$",
            r"^sm__instruction_throughput\.avg\.pct_of_peak_sustained_active$", r"^l1tex__throughput\.avg\.pct_of_peak_sustained_active$"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_tc.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "launch__shared_mem_per_block_dynamic", "lts__t_bytes.sum", "l1tex__t_bytes.sum",
    "smsp__inst_executed.sum", "sm__cycles_elapsed.avg",
]


def short(name):
    name = name.split("(")[0]
    for p in ("void ", "psim::"):
        name = name.replace(p, "")
    return name.strip()


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[hdr_i]
    kn, mn, mv, un = (hdr.index(x) for x in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[hdr_i + 1:]:
        if len(r) <= mv or r[mn] != "gpu__time_duration.sum":
            continue
        v = float(r[mv].replace(",", ""))
        unit = r[un]
        ns = v * {"nsecond": 1, "usecond": 1e3, "msecond": 1e6, "second": 1e9}.get(unit, 1)
        a = agg[short(r[kn])]
        a[0] += 1
        a[1] += ns
    tot = sum(a[1] for a in agg.values())
    lines = ["| kernel | launches | total ms | mean us | share |", "|---|---|---|---|---|"]
    for k, (c, ns) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        lines.append(f"| `{k}` | {c} | {ns / 1e6:.3f} | {ns / c / 1e3:.2f} | {ns / tot:.3f} |")
    return "\n".join(lines), agg


def rep(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": short(dict(zip(hdr, r)).get("Kernel Name", "?")), "metrics": {}}
        for k, u, v in zip(hdr, units, r):
            if any(re.search(p, k) for p in PATTERNS) and v != "":
                if "tensor" in k and (re.search(r"\.(max|min|sum)\.pct", k) or v.strip() in ("0", "0.000000")):
                    continue
                d["metrics"][k] = (v, u)
        rd = d["metrics"].get("dram__bytes_read.sum"), d["metrics"].get("dram__bytes_write.sum")
        if all(rd):
            d["dram_bytes"] = sum(float(v.replace(",", "")) * SCALE.get(u, 1) for v, u in rd)
        res.append(d)
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--rep")
    ap.add_argument("--out", required=True)
    ap.add_argument("--title", default="")
    ap.add_argument("--traffic-key")
    a = ap.parse_args()
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    text = [f"# {a.title or os.path.basename(a.out)}", ""]
    if a.launches:
        t, _ = launches(a.launches)
        text += [f"Source: `{a.launches}` (ncu --metrics gpu__time_duration.sum --clock-control none)", "", t]
    if a.rep:
        res = rep(a.rep)
        text += [f"Source: `{a.rep}` (ncu --set full --clock-control none)", ""]
        for i, d in enumerate(res):
            text.append(f"## launch {i}: `{d['kernel']}`")
            for k, (v, u) in sorted(d["metrics"].items()):
                text.append(f"- {k}: {v} {u}")
            if "dram_bytes" in d:
                text.append(f"- DRAM bytes (read + write): {d['dram_bytes']:.4g}")
            text.append("")
        if a.traffic_key and res:
            per = [d.get("dram_bytes", 0.0) for d in res]
            tj = "profiles/ncu_traffic.json"
            cur = json.load(open(tj)) if os.path.exists(tj) else {}
            cur[a.traffic_key] = {"dram_bytes_per_launch": sum(per) / len(per), "source": a.rep,
                                  "launches": len(per)}
            json.dump(cur, open(tj, "w"), indent=1)
    open(a.out, "w").write("\n".join(text) + "\n")
    print("\n".join(text))


if __name__ == "__main__":
    main()
