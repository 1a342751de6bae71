#!/usr/bin/env python
"""Decode an MBIR_TRACE dump (per-pair clock64 stamps of one SV visit of CTA 0; DESIGN.md s.11).
Columns (cycles, relative to the pair's gather start on view warp 0)."""
import sys
import numpy as np
t = np.fromfile(sys.argv[1], dtype=np.uint64).astype(np.int64)
nact = int(t[0]) - 1
T = t[1:1009].reshape(-1, 16)
task = T[60]
print(f"nact {nact}  visit: order {task[1]-task[0]}  pack {task[2]-task[1]}  loop {task[3]-task[2]}  writeback {task[4]-task[3]}")
names = {0: "v0 gather", 1: "v0 arriveA", 2: "v0 prep done", 3: "v0 B woke", 4: "v0 scatter done",
         8: "v5 gather", 9: "v5 arriveA", 10: "v5 prep done", 11: "v5 B woke", 12: "v5 scatter done",
         5: "pri wait A", 6: "pri A woke", 7: "pri publish", 13: "pri next terms"}
npair = (nact + 1) // 2
rows = []
for p in range(npair):
    r = T[p]
    base = r[0]
    rows.append({k: int(r[k] - base) for k in names})
    if p < 6 or p == npair - 1:
        print(f"pair {p:2d} period {int(T[p+1][0]-r[0]) if p+1 < npair else 0:6d} | " +
              " ".join(f"{names[k]}={int(r[k]-base)}" for k in sorted(names)))
import statistics as st
mid = rows[2:npair - 2]
print("median over pairs:")
for k in sorted(names):
    print(f"  {names[k]:16s} {st.median(r[k] for r in mid):8.0f}")
per = [int(T[p + 1][0] - T[p][0]) for p in range(2, npair - 2)]
print("median pair period", st.median(per))
