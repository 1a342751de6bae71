#!/usr/bin/env python
"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list: per-kernel count,
total device time and share.  Usage: tools/launch_summary.py launches.csv"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
hdr = rows[start]
ik, iv, iu = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
tot, cnt = collections.defaultdict(float), collections.Counter()
for r in rows[start + 1:]:
    if len(r) <= iv:
        continue
    name = r[ik].split("(")[0].replace("void ", "").strip().split("::")[-1]
    v = float(r[iv].replace(",", ""))
    v *= {"usecond": 1e3, "msecond": 1e6}.get(r[iu], 1.0)
    tot[name] += v
    cnt[name] += 1
T = sum(tot.values())
print(f"{'kernel':40s} {'launches':>8s} {'total ms':>10s} {'share':>7s}")
for k, v in sorted(tot.items(), key=lambda x: -x[1]):
    print(f"{k:40s} {cnt[k]:8d} {v / 1e6:10.3f} {100 * v / T:6.2f}%")
