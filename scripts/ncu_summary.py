#!/usr/bin/env python
"""Summarise ncu artefacts from gpurun_out/ into profiles/ (committed).

    python scripts/ncu_summary.py TAG WORKLOAD [--rep gpurun_out/prof_TAG_WL.ncu-rep]
                                               [--launches gpurun_out/launches_TAG_WL.csv]

Writes profiles/ncu_TAG_WL.md (human readable) and merges the per-kernel
numbers into profiles/ncu_summary.json (read by bench.py for `traffic`).
"""
import argparse
import csv
import io
import json
import os
import subprocess
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "lts__t_bytes.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "l1tex__throughput.avg.pct_of_peak_sustained_active",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
    "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum",
    "smsp__thread_inst_executed_per_inst_executed.ratio", "sm__cycles_active.avg",
    "sm__cycles_active.max", "gpc__cycles_elapsed.max", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "lts__t_sector_hit_rate.pct", "smsp__warps_eligible.avg.per_cycle_active",
]


def short(name):
    import re
    m = re.search(r"(list_(?:warp|block)_kernel)<(true|false|1|0)", name)
    if m:
        return f"{m.group(1)}<{'tri' if m.group(2) in ('true', '1') else 'support'}>"
    m = re.search(r"support_hash_kernel<\d+>", name)
    if m:
        return m.group(0)
    for k in ("support_kernel", "edge_fc_kernel", "tri_core_kernel", "vertex_core_kernel", "core_kernel"):
        if k in name:
            return k
    return name.split("(")[0][-40:]


def raw_page(rep):
    """rows of the raw page: from an .ncu-rep (via ncu -i) or from its
    exported CSV (ncu -i REP --page raw --csv > X_raw.csv, done on the GPU box
    so the large report need not travel back)"""
    if rep.endswith(".csv"):
        out = open(rep).read()
    else:
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        d["_units"] = dict(zip(hdr, units))
        res.append(d)
    return res


SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}


def to_bytes(d, m):
    v = num(d.get(m))
    u = d["_units"].get(m, "byte")
    return None if v is None else v * SCALE.get(u, 1)


def num(x):
    try:
        return float(str(x).replace(",", ""))
    except ValueError:
        return None


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hdr]
    ki, vi = h.index("Kernel Name"), h.index("Metric Value")
    agg = defaultdict(list)
    for r in rows[hdr + 1:]:
        agg[short(r[ki])].append(num(r[vi]))
    return agg


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("tag")
    ap.add_argument("workload")
    ap.add_argument("--rep")
    ap.add_argument("--launches")
    a = ap.parse_args()
    rep = a.rep or os.path.join(ROOT, "gpurun_out", f"prof_{a.tag}_{a.workload}.ncu-rep")
    if not os.path.exists(rep) and os.path.exists(rep.replace(".ncu-rep", "_raw.csv")):
        rep = rep.replace(".ncu-rep", "_raw.csv")
    lpath = a.launches or os.path.join(ROOT, "gpurun_out", f"launches_{a.tag}_{a.workload}.csv")
    md = [f"# ncu summary {a.tag} / {a.workload}", ""]
    kern = {}
    if os.path.exists(rep):
        md += ["## `ncu --set full` capture (one launch per kernel, cold caches, clocks not locked)", "",
               "| kernel | " + " | ".join(m.split("__")[1] if "__" in m else m for m in METRICS) + " |",
               "|---" * (len(METRICS) + 1) + "|"]
        for d in raw_page(rep):
            k = short(d.get("Kernel Name", "?"))
            vals = [d.get(m, "") for m in METRICS]
            md.append(f"| {k} | " + " | ".join(str(v) for v in vals) + " |")
            rd, wr = to_bytes(d, "dram__bytes_read.sum"), to_bytes(d, "dram__bytes_write.sum")
            kern[k] = {m: (d.get(m), d["_units"].get(m)) for m in METRICS}
            kern[k]["dram_bytes_per_launch"] = (rd or 0) + (wr or 0)
        md.append("")
        md.append("(units as ncu prints them in the raw page; `dram__bytes_*` are per launch)")
        md += ["", "### warp stall reasons (PC sampling, top 6 per kernel)", ""]
        for d in raw_page(rep):
            st = []
            for h, v in d.items():
                if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("not_issued"):
                    x = num(v)
                    if x:
                        st.append((x, h.replace("smsp__pcsamp_warps_issue_stalled_", "")))
            st.sort(reverse=True)
            tot = sum(x for x, _ in st) or 1.0
            md.append(f"- {short(d.get('Kernel Name', '?'))}: " +
                      ", ".join(f"{h} {100 * x / tot:.0f}%" for x, h in st[:6]))
    if os.path.exists(lpath):
        agg = launches(lpath)
        tot = sum(sum(v) for v in agg.values())
        md += ["", "## launch list (`--metrics gpu__time_duration.sum`, serialized, cold)", "",
               "| kernel | launches | mean ns | share of listed time |", "|---|---|---|---|"]
        for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
            md.append(f"| {k} | {len(v)} | {sum(v) / len(v):.0f} | {sum(v) / tot:.3f} |")
    out_md = os.path.join(ROOT, "profiles", f"ncu_{a.tag}_{a.workload}.md")
    os.makedirs(os.path.dirname(out_md), exist_ok=True)
    open(out_md, "w").write("\n".join(md) + "\n")
    sj = os.path.join(ROOT, "profiles", "ncu_summary.json")
    summary = json.load(open(sj)) if os.path.exists(sj) else {}
    summary.setdefault(a.workload, {})
    summary[a.workload]["tag"] = a.tag
    summary[a.workload]["kernels"] = kern
    json.dump(summary, open(sj, "w"), indent=1)
    print(open(out_md).read())


if __name__ == "__main__":
    main()
