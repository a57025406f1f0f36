#!/usr/bin/env python
"""Aggregate an ncu --csv launch list (gpu__time_duration.sum) by kernel."""
import csv
import io
import sys
txt = open(sys.argv[1]).read().splitlines()
i = next(k for k, ln in enumerate(txt) if ln.startswith('"ID"'))
rows = [r for r in csv.DictReader(io.StringIO("\n".join(txt[i:]))) if r.get("Metric Name") == "gpu__time_duration.sum"]
agg = {}
for r in rows:
    agg.setdefault(r["Kernel Name"][:80], []).append(float(r["Metric Value"]))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 10
for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1]))[:top]:
    print(f"{len(v):4d} x {sum(v) / len(v) / 1e3:10.1f} us  {k}")
