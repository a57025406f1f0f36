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

# all rows as (offset from the function's first instruction, samples, warp
# instructions executed) for local mapping to source lines (nvdisasm -g)
if len(sys.argv) > 3:
    addr = [int(r[col["Address"]], 16) for _, r in data]
    base = min(addr) if addr else 0
    ie = col.get("Instructions Executed")
    with open(sys.argv[3], "w") as f:
        for (v, r), a in zip(data, addr):
            x = r[ie].replace(",", "") if ie is not None else "0"
            if v or (x not in ("", "0")):
                f.write(f"{a - base},{v:.0f},{x}\n")
