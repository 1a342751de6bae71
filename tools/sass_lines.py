#!/usr/bin/env python
"""Aggregate an ncu SASS source page (csv) by CUDA source line, using nvdisasm -gi line info of
the same cubin.  usage: sass_lines.py <ncu-rep> <cubin> <function-substring> [top]"""
import csv
import io
import re
import subprocess
import sys

rep, cubin, fsub = sys.argv[1:4]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
dis = subprocess.run(["nvdisasm", "-gi", cubin], capture_output=True, text=True).stdout
addr2line, cur_fn, line = {}, None, None
for ln in dis.splitlines():
    m = re.match(r"\s*\.text\.(\S+):", ln)
    if m:
        cur_fn = m.group(1)
        continue
    if cur_fn is None or fsub not in cur_fn:
        continue
    m = re.search(r'line (\d+)(?: inlined at .*line (\d+))?', ln)
    if "//##" in ln and m:
        line = int(m.group(2) or m.group(1))
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", ln)
    if m and line is not None:
        addr2line[int(m.group(1), 16)] = line
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = next(r for r in rows if r and r[0] == "Address")
body = rows[rows.index(hdr) + 1:]
ix = hdr.index("Warp Stall Sampling (All Samples)")
ex = hdr.index("Instructions Executed")
stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
agg = {}
tot = 0.0
base = None
for r in body:
    if len(r) <= ix or not r[0].startswith("0x"):
        continue
    a = int(r[0], 16)
    base = a if base is None else base
    a -= base
    s = float(r[ix] or 0)
    tot += s
    L = addr2line.get(a, -1)
    d = agg.setdefault(L, [0.0, 0.0, {}])
    d[0] += s
    d[1] += float(r[ex] or 0)
    for c in stall_cols:
        v = float(r[c] or 0)
        if v:
            d[2][hdr[c]] = d[2].get(hdr[c], 0) + v
print(f"total samples {tot:.0f}; mapped lines {len(agg)}")
for L, (s, e, st) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    top3 = sorted(st.items(), key=lambda kv: -kv[1])[:3]
    print(f"{100 * s / tot:5.1f}%  L{L:<5d} inst {e:12.0f}  " + " ".join(f"{k[6:]}:{100 * v / tot:.1f}" for k, v in top3))
