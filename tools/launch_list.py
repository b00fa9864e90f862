"""One bench-configuration training step between cudaProfilerStart/Stop, for
`ncu --profile-from-start off --metrics gpu__time_duration.sum` launch lists.
    python tools/launch_list.py [workload] [budget_frac] [eager|graph]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen  # noqa: E402

wl = sys.argv[1] if len(sys.argv) > 1 else "bert_large"
frac = float(sys.argv[2]) if len(sys.argv) > 2 else bench.WORKLOADS[wl]["frac"]
mode = sys.argv[3] if len(sys.argv) > 3 else "graph"
spec = bench.workload_graph(wl)
G = tsplit.Graph(spec)
st = tsplit.Plan.default(G).stats()
budget = st["static_bytes"] + int(frac * (st["peak_extent"] - st["static_bytes"]))
dev = tsplit.inputs_to_device(G, gen.make_inputs(spec))
prof = tsplit.Profile.measure(G, dev, max_p=16)
P = tsplit.Plan.plan(G, budget, prof)
S = tsplit.Session(G, P, lr=1e-4, use_cuda_graph=(mode == "graph"))
S.set_params(gen.init_params(spec))
for _ in range(2):
    S.step(dev)
torch.cuda.synchronize()
torch.cuda.profiler.start()
S.step(dev)
torch.cuda.synchronize()
torch.cuda.profiler.stop()
print("kernels per step", S.launches())
