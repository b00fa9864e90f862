"""Aggregate an ncu --csv launch list (gpu__time_duration.sum) by kernel name.
    python tools/summarize_launches.py launches.csv [out.csv]"""
import collections
import csv
import re
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hdr_i]
ik, iv, im = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Name")
agg = collections.defaultdict(lambda: [0, 0.0])
for r in rows[hdr_i + 1:]:
    if len(r) <= iv or r[im] != "gpu__time_duration.sum":
        continue
    name = re.sub(r"\(.*", "", r[ik]).replace("void ", "").strip()
    v = float(r[iv].replace(",", ""))
    unit = r[h.index("Metric Unit")] if "Metric Unit" in h else "ns"
    us = v / 1e3 if unit in ("nsecond", "ns") else (v if unit in ("usecond", "us") else v * 1e3)
    agg[name][0] += 1
    agg[name][1] += us
tot = sum(v[1] for v in agg.values())
out = [("kernel", "launches", "total_us", "share")]
for k, (n, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    out.append((k, n, round(us, 1), round(us / tot, 4)))
for r in out[:30]:
    print(*r, sep="\t")
print("total_us", round(tot, 1))
if len(sys.argv) > 2:
    csv.writer(open(sys.argv[2], "w")).writerows(out)
