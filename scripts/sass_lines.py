#!/usr/bin/env python
"""Aggregate an ncu per-offset export (src_hot.py's third argument) by CUDA
source line, using `nvdisasm -g -c` line info of the same cubin:
    python scripts/sass_lines.py DISASM.sass KERNEL_SUBSTR OFFS.csv [N]"""
import collections
import re
import sys

sass, kname, offs = sys.argv[1], sys.argv[2], sys.argv[3]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
line_of = {}
cur_line, inside = None, False
for ln in open(sass, errors="replace"):
    if ln.startswith(".text."):
        inside = kname in ln
        continue
    if not inside:
        continue
    m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
    if m:
        f = m.group(1).split("/")[-1]
        inl = re.search(r'inlined at "([^"]+)", line (\d+)', ln)
        cur_line = f"{f}:{m.group(2)}" + (f" (in {inl.group(1).split('/')[-1]}:{inl.group(2)})" if inl else "")
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", ln)
    if m:
        line_of[int(m.group(1), 16)] = cur_line
samp, inst = collections.Counter(), collections.Counter()
for row in open(offs):
    o, s, x = row.strip().split(",")
    k = line_of.get(int(o), "?")
    samp[k] += float(s)
    inst[k] += float(x or 0)
ts, ti = sum(samp.values()) or 1, sum(inst.values()) or 1
print(f"# total samples {ts:.0f}, warp instructions {ti:.3g}")
for k, v in samp.most_common(top):
    print(f"{100 * v / ts:6.2f}% samples {100 * inst[k] / ti:6.2f}% inst  {k}")
