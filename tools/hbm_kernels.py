"""Per-kernel HBM throughput from an ncu --csv capture with gpu__time_duration.sum,
dram__bytes_read.sum and dram__bytes_write.sum (one eager step, tools/step_once.py):
for every kernel name, launches, total time, DRAM bytes, achieved GB/s and the fraction
of MEASURED_PEAKS.json hbm_gbs.  python tools/hbm_kernels.py capture.csv [out.json]"""
import collections
import csv
import json
import os
import re
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hdr_i]
ik, iv, im, iid = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Name"), h.index("ID")
iu = h.index("Metric Unit") if "Metric Unit" in h else None
per = collections.defaultdict(dict)
names = {}
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3,
         "ns": 1e-9, "us": 1e-6, "ms": 1e-3}
for r in rows[hdr_i + 1:]:
    if len(r) <= iv:
        continue
    unit = r[iu] if iu is not None else ""
    v = float(r[iv].replace(",", "")) * scale.get(unit, 1.0)
    per[r[iid]][r[im]] = v
    names[r[iid]] = re.sub(r"\(.*", "", r[ik]).replace("void ", "").strip()
peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                   "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6554.9
agg = collections.defaultdict(lambda: [0, 0.0, 0.0])
for lid, m in per.items():
    a = agg[names[lid]]
    a[0] += 1
    a[1] += m.get("gpu__time_duration.sum", 0.0)
    a[2] += m.get("dram__bytes_read.sum", 0.0) + m.get("dram__bytes_write.sum", 0.0)
tot = sum(a[1] for a in agg.values())
out = []
for k, (n, t, b) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    out.append({"kernel": k, "launches": n, "total_us": round(t * 1e6, 1), "share": round(t / tot, 4),
                "dram_bytes": int(b), "achieved_gbs": round(b / t / 1e9, 1) if t else None,
                "frac_of_hbm_peak": round(b / t / 1e9 / peak, 3) if t else None})
for r in out[:25]:
    print(r)
if len(sys.argv) > 2:
    json.dump({"hbm_peak_gbs": peak, "how": "ncu --clock-control none, one eager step (cold-cache, serialised "
               "launches): dram read+write bytes / gpu__time_duration per kernel name", "kernels": out},
              open(sys.argv[2], "w"), indent=1)
