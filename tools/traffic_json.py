#!/usr/bin/env python
"""profiles/icd_traffic.json from a tools/traffic.sh capture: ncu DRAM bytes of every k_svicd
launch of one bench step / that step's executed voxel updates.  usage: traffic_json.py PREFIX"""
import csv
import json
import sys

pre = sys.argv[1]
rows = [r for r in csv.reader(open(pre + ".csv")) if len(r) > 10]
h = rows[0]
im, iv, iu = h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
tot, launches = {}, set()
for r in rows[1:]:
    tot[r[im]] = tot.get(r[im], 0.0) + float(r[iv].replace(",", "")) * scale.get(r[iu], 1.0)
    launches.add(r[0])
line = next(ln for ln in open(pre + ".json") if ln.startswith("{"))
upd = json.loads(line)["updates_per_step"]
out = {
    "dram_bytes_per_update": round((tot["dram__bytes_read.sum"] + tot["dram__bytes_write.sum"]) / upd, 1),
    "dram_read_bytes_per_update": round(tot["dram__bytes_read.sum"] / upd, 1),
    "dram_write_bytes_per_update": round(tot["dram__bytes_write.sum"] / upd, 1),
    "l2_bytes_per_update": round(tot["lts__t_bytes.sum"] / upd, 1),
    "launches": len(launches),
    "updates": upd,
    "how": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum over every k_svicd "
           "launch of one bench.py step (cfg4, 6 equits from x0 = 0; tools/traffic.sh)",
}
print(json.dumps(out, indent=1))
