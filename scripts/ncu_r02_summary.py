#!/usr/bin/env python
"""Merge an ncu raw-page CSV export (gpurun_out/prof_TAG_WL_raw.csv, or a
--metrics launch CSV) into profiles/ncu_r02_summary.json, per workload and
kernel (short name, e.g. list_block_kernel<tri-z>), per launch:
    python scripts/ncu_r02_summary.py TAG WORKLOAD RAW.csv
bench.py reads `dram_bytes_per_launch` (roofline.traffic) and
`inst_per_launch` (issue-rate roofline of the listing kernels) from it."""
import csv
import json
import os
import re
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "profiles", "ncu_r02_summary.json")
MODES = {"0": "support", "1": "tri", "2": "tri-z"}
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ns": 1e-9, "us": 1e-6, "usecond": 1e-6,
         "ms": 1e-3, "msecond": 1e-3, "s": 1.0, "second": 1.0, "nsecond": 1e-9, "inst": 1, "": 1,
         "Kinst": 1e3, "Minst": 1e6, "Ginst": 1e9}


def short(name):
    m = re.search(r"(list_(?:warp|block)_kernel)<(\d)", name)
    if m:
        return f"{m.group(1)}<{MODES.get(m.group(2), m.group(2))}>"
    for k in ("support_kernel", "edge_fc_kernel", "vertex_core_kernel", "core_kernel"):
        if k in name:
            return k
    return name.split("(")[0][-40:]


def main():
    tag, wl, path = sys.argv[1], sys.argv[2], sys.argv[3]
    txt = open(path).read()
    if '"Metric Name"' in txt:          # --metrics --csv (long format): pivot to one row per launch
        import io
        body = txt[txt.index('"ID"'):]
        lr = list(csv.reader(io.StringIO(body)))
        hc = {c: i for i, c in enumerate(lr[0])}
        launches, order, mets, munit = {}, [], [], {}
        for r in lr[1:]:
            if len(r) < len(lr[0]):
                continue
            key = r[hc["ID"]]
            if key not in launches:
                launches[key] = {"Kernel Name": r[hc["Kernel Name"]]}
                order.append(key)
            mn = r[hc["Metric Name"]]
            launches[key][mn] = r[hc["Metric Value"]]
            munit[mn] = r[hc["Metric Unit"]]
            if mn not in mets:
                mets.append(mn)
        h = ["Kernel Name"] + mets
        rows = [h, [""] + [munit[m] for m in mets]] + [[launches[k].get(c, "") for c in h] for k in order]
    else:
        rows = list(csv.reader(io.StringIO(txt))) if False else list(csv.reader(open(path)))
        h = rows[0]
    units = rows[1]
    col = {c: i for i, c in enumerate(h)}
    name_col = col.get("Kernel Name")
    acc = defaultdict(lambda: defaultdict(float))
    cnt = defaultdict(int)
    for r in rows[2:]:
        if len(r) < len(h):
            continue
        k = short(r[name_col])
        cnt[k] += 1
        for metric, key in (("gpu__time_duration.sum", "time_s"), ("dram__bytes_read.sum", "dram_read"),
                            ("dram__bytes_write.sum", "dram_write"), ("smsp__inst_executed.sum", "inst"),
                            ("lts__t_bytes.sum", "l2_bytes")):
            if metric in col:
                v = r[col[metric]].replace(",", "")
                try:
                    acc[k][key] += float(v) * SCALE.get(units[col[metric]], 1)
                except ValueError:
                    pass
    d = json.load(open(OUT)) if os.path.exists(OUT) else {}
    ent = d.setdefault(wl, {"tag": tag, "kernels": {}})
    ent["tag"] = tag
    for k, v in acc.items():
        n = cnt[k]
        ent["kernels"][k] = {"launches": n, "time_s_per_launch": v["time_s"] / n,
                             "dram_bytes_per_launch": (v["dram_read"] + v["dram_write"]) / n,
                             "l2_bytes_per_launch": v["l2_bytes"] / n if v["l2_bytes"] else None,
                             "inst_per_launch": v["inst"] / n if v["inst"] else None, "source": os.path.basename(path)}
    json.dump(d, open(OUT, "w"), indent=1, sort_keys=True)
    print(json.dumps(ent, indent=1))


if __name__ == "__main__":
    main()
