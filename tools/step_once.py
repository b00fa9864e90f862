"""One eager BERT step between cudaProfilerStart/Stop (all-reside plan unless a budget
fraction is given), for ncu captures of in-step kernels:
    python tools/step_once.py [layers] [budget_frac]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402

layers = int(sys.argv[1]) if len(sys.argv) > 1 else 2
frac = float(sys.argv[2]) if len(sys.argv) > 2 else 0.0
spec = graphs.bert(layers=layers, batch=32, fused_attention=True)
G = tsplit.Graph(spec)
P = tsplit.Plan.default(G)
if frac > 0:
    st = P.stats()
    P = tsplit.Plan.plan(G, st["static_bytes"] + int(frac * (st["peak_extent"] - st["static_bytes"])))
S = tsplit.Session(G, P, lr=1e-4, use_cuda_graph=False)
S.set_params(gen.init_params(spec))
dev = tsplit.inputs_to_device(G, gen.make_inputs(spec))
S.step(dev)
torch.cuda.synchronize()
torch.cuda.profiler.start()
S.step(dev)
torch.cuda.synchronize()
torch.cuda.profiler.stop()
print("kernels per step", S.launches())
