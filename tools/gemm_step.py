"""Per-GEMM-shape in-step throughput of one BERT-Large step (eager, profiled):
groups the session's GEMM/conv records by (kind, M, N, K, batch).
    python tools/gemm_step.py [fused|unfused] [budget_frac or 0 for all-reside]"""
import collections
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402

fused = len(sys.argv) < 2 or sys.argv[1] == "fused"
frac = float(sys.argv[2]) if len(sys.argv) > 2 else 0.0
tsplit.check(tsplit.lib().ts_gemm_set_mode(int(os.environ.get("GEMM_MODE", "0"))))
spec = graphs.bert(layers=24, batch=32, fused_attention=fused)
G = tsplit.Graph(spec)
P = tsplit.Plan.default(G)
if frac > 0:
    st = P.stats()
    P = tsplit.Plan.plan(G, st["static_bytes"] + int(frac * (st["peak_extent"] - st["static_bytes"])))
S = tsplit.Session(G, P, lr=1e-4)
S.set_params(gen.init_params(spec))
dev = tsplit.inputs_to_device(G, gen.make_inputs(spec))
S.step(dev)
S.profile_items(True)
S.step(dev)
recs = S.gemm_times()
kinds = S.gemm_kinds()
shapes = S.gemm_shapes()
lib = tsplit.lib()
import ctypes as C  # noqa: E402
n = C.c_uint64()
# shapes are not exposed per record; rebuild them from the GemmRecord order via flop and batch
agg = collections.defaultdict(lambda: [0, 0.0, 0.0])
for (f, ms, bt), (kd, tc), sh in zip(recs, kinds, shapes):
    key = (kd, bt, sh, tc)
    a = agg[key]
    a[0] += 1
    a[1] += ms
    a[2] += f
tot_ms = sum(v[1] for v in agg.values())
print(f"GEMM launches {len(recs)}  total {tot_ms:.2f} ms  avg {sum(v[2] for v in agg.values()) / tot_ms / 1e9:.0f} TFLOP/s")
for key, (cnt, ms, f) in sorted(agg.items(), key=lambda kv: -kv[1][1])[:25]:
    print(f"kind {key[0]} batch {key[1]:4d} MNK,flags {str(key[2]):28s} tc {key[3]}  n={cnt:4d}  {ms:8.2f} ms  "
          f"{f / ms / 1e9:7.0f} TFLOP/s  {ms / cnt * 1e3:7.1f} us/launch")

del S, P, G
