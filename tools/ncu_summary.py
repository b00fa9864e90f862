"""Summarise one kernel of an ncu --set full report into the JSON kept under profiles/.
    python tools/ncu_summary.py report.ncu-rep kernel_regex "description" out.json [algorithmic_bytes]"""
import csv
import io
import json
import re
import subprocess
import sys

rep, kre, desc, out = sys.argv[1:5]
alg = float(sys.argv[5]) if len(sys.argv) > 5 else None
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h = rows[0]
d = next(dict(zip(h, r)) for r in rows[2:] if re.search(kre, r[h.index("Kernel Name")]))
f = lambda k: float(d[k].replace(",", "")) if d.get(k) not in (None, "") else None  # noqa: E731
res = {
    "kernel": d["Kernel Name"][:160],
    "source": desc,
    "duration_us_under_ncu": f("gpu__time_duration.sum"),
    "dram_bytes_read": f("dram__bytes_read.sum"),
    "dram_bytes_write": f("dram__bytes_write.sum"),
    "tensor_pipe_active_pct": f("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active"),
    "sm_throughput_pct": f("sm__throughput.avg.pct_of_peak_sustained_elapsed"),
    "dram_throughput_pct": f("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"),
}
units = {k: d.get(k) for k in ("dram__bytes_read.sum", "dram__bytes_write.sum")}
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
u = rows[1][h.index("dram__bytes_read.sum")]
for k in ("dram_bytes_read", "dram_bytes_write"):
    if res[k] is not None:
        res[k] *= scale.get(u, 1)
res["traffic_per_launch_bytes"] = (res["dram_bytes_read"] or 0) + (res["dram_bytes_write"] or 0)
if alg:
    res["algorithmic_bytes"] = alg
json.dump(res, open(out, "w"), indent=1)
print(json.dumps(res, indent=1))
