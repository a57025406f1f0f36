#!/usr/bin/env python
"""Summarise one round-2 measurement into profiles/ (committed evidence):
    python scripts/profile_md.py TAG WORKLOAD
reads gpurun_out/ncum_TAG_WORKLOAD.csv (ncu --metrics, long format),
gpurun_out/launches_TAG_WORKLOAD.csv (ncu launch list of the bench command)
and gpurun_out/bench_TAG.json; writes profiles/ncu_TAG_WORKLOAD.md and copies
the bench line to profiles/bench_TAG_WORKLOAD.json."""
import csv
import io
import json
import os
import re
import shutil
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag, wl = sys.argv[1], sys.argv[2]
G = os.path.join(ROOT, "gpurun_out")
out = [f"# ncu summary {tag}, workload {wl}", ""]


def long_rows(path):
    txt = open(path).read()
    body = txt[txt.index('"ID"'):]
    return list(csv.reader(io.StringIO(body)))


def short(name):
    m = re.search(r"(list_(?:warp|block)_kernel)<(\d)", name)
    if m:
        return f"{m.group(1)}<{ {'0': 'support', '1': 'tri', '2': 'tri-z'}[m.group(2)] }>"
    return re.sub(r"\(.*", "", name).replace("void ", "").replace("<unnamed>::", "")[:60]


p = os.path.join(G, f"ncum_{tag}_{wl}.csv")
if os.path.exists(p):
    rows = long_rows(p)
    h = {c: i for i, c in enumerate(rows[0])}
    per = defaultdict(dict)
    for r in rows[1:]:
        if len(r) < len(rows[0]):
            continue
        per[(r[h["ID"]], short(r[h["Kernel Name"]]))][r[h["Metric Name"]]] = (r[h["Metric Value"]], r[h["Metric Unit"]])
    mets = sorted({m for d in per.values() for m in d})
    out += ["## Per-kernel metrics (`ncu --metrics`, one launch each, clocks not locked)", "",
            "| kernel | " + " | ".join(mets) + " |", "|---|" + "---|" * len(mets)]
    for (i, k), d in per.items():
        out.append(f"| {k} | " + " | ".join(f"{d[m][0]} {d[m][1]}" if m in d else "" for m in mets) + " |")
    out.append("")
p = os.path.join(G, f"launches_{tag}_{wl}.csv")
if os.path.exists(p):
    rows = long_rows(p)
    h = {c: i for i, c in enumerate(rows[0])}
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[1:]:
        if len(r) < len(rows[0]) or r[h["Metric Name"]] != "gpu__time_duration.sum":
            continue
        v = float(r[h["Metric Value"]].replace(",", ""))
        unit = r[h["Metric Unit"]]
        v *= {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0, "s": 1e3, "second": 1e3,
              "nsecond": 1e-6}.get(unit, 1.0)
        k = short(r[h["Kernel Name"]])
        agg[k][0] += 1
        agg[k][1] += v
    tot = sum(v for _, v in agg.values()) or 1.0
    out += ["## Launch list of the bench command (`ncu --metrics gpu__time_duration.sum`, serialised, cold caches)",
            "", "| kernel | launches | total ms | share |", "|---|---|---|---|"]
    for k, (n, v) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        out.append(f"| {k} | {n} | {v:.2f} | {100 * v / tot:.1f} % |")
    out.append("")
p = os.path.join(G, f"bench_{tag}.json")
if os.path.exists(p):
    line = json.loads([ln for ln in open(p) if ln.startswith("{")][0])
    shutil.copy(p, os.path.join(ROOT, "profiles", f"bench_{tag}_{wl}.json"))
    rf = line["roofline"]
    out += ["## Bench line (device-timed, L2 flushed per step)", "",
            f"- value {line['value']:.4g} {line['unit']}, {line['ms_per_step']:.1f} ms/step, "
            f"edges/s {line.get('edges_per_s', 0):.4g}, clocks {line.get('clocks')}",
            f"- dominant kernel: {rf['kernel']}: {rf['kernel_ms']:.1f} ms ({100 * rf['share_of_step']:.1f} % of the step), "
            f"bound {rf['bound']}, achieved {rf['achieved']:.4g} / peak {rf['peak']:.4g} {rf['unit']} = frac {rf['frac']:.3f}, "
            f"traffic {rf.get('traffic')}",
            ]
    for o in line.get("roofline_other_kernels", []):
        out.append(f"- {o['kernel']}: {o['kernel_ms']:.1f} ms, bound {o['bound']}, frac {o['frac']:.3f}, traffic {o.get('traffic')}")
    if line.get("e2e"):
        out.append(f"- e2e: {line['e2e']}")
    if line.get("cpu_baseline"):
        out.append(f"- cpu_baseline: {line['cpu_baseline']}")
open(os.path.join(ROOT, "profiles", f"ncu_{tag}_{wl}.md"), "w").write("\n".join(out) + "\n")
print("\n".join(out))
