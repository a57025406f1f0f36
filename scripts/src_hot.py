#!/usr/bin/env python
"""Hottest SASS lines of an `ncu --page source --csv` export (by warp stall
samples), with their CUDA source location: python scripts/src_hot.py X.csv [N]"""
import csv
import sys

path = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 60
rows = list(csv.reader(open(path, errors="replace")))
hdr_i = next((i for i, r in enumerate(rows) if any("Sampling" in c for c in r)), None)
if hdr_i is None:
    print("no source page rows"); sys.exit(0)
h = rows[hdr_i]
col = {c: i for i, c in enumerate(h)}
samp = next(c for c in h if c.startswith("Warp Stall Sampling (All"))
data = []
for r in rows[hdr_i + 1:]:
    if len(r) < len(h):
        continue
    try:
        v = float(r[col[samp]].replace(",", "") or 0)
    except ValueError:
        continue
    data.append((v, r))
tot = sum(v for v, _ in data) or 1.0
print(f"# {path}: {len(data)} rows, total samples {tot:.0f}; columns: {h[:12]}")
data.sort(key=lambda x: -x[0])
for v, r in data[:top]:
    print(f"{100 * v / tot:6.2f}%  " + " | ".join(x.strip()[:90] for x in r[:4]))
