"""Trial-time the planner variants on one workload (measured / analytic profile x default /
w/o split / memory-centric), each 2 warm-up + 3 timed steps.
    python tools/plan_variants.py [bert_large|vgg16|resnet50]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen  # noqa: E402

wl = sys.argv[1] if len(sys.argv) > 1 else "resnet50"
W = bench.WORKLOADS[wl]
spec = bench.workload_graph(wl)
G = tsplit.Graph(spec)
st = tsplit.Plan.default(G).stats()
budget = st["static_bytes"] + int(W["frac"] * (st["peak_extent"] - st["static_bytes"]))
dev = tsplit.inputs_to_device(G, gen.make_inputs(spec))
prof = tsplit.Profile.measure(G, dev, max_p=16)
params = gen.init_params(spec, seed=1)
out = {}
for pname, pr in (("measured", prof), ("analytic", None)):
    for vname, kw in (("default", {}), ("no_split", {"no_split": True}), ("memory_centric", {"memory_centric": True})):
        key = f"{pname}/{vname}"
        try:
            P = tsplit.Plan.plan(G, budget, pr, **kw)
        except tsplit.TsError as e:
            out[key] = f"infeasible: {str(e)[:60]}"
            print(key, out[key], flush=True)
            continue
        stream = torch.cuda.Stream()
        S = tsplit.Session(G, P, lr=1e-4, streams=(stream, torch.cuda.Stream(), torch.cuda.Stream()))
        S.set_params(params)
        for _ in range(2):
            S.step(dev)
        ms = bench.time_steps(torch, S, dev, stream, 3) / 3 * 1e3
        s = P.stats()
        out[key] = {"ms": round(ms, 2), "pred_ms": round(s["predicted_s"] * 1e3, 2), "splits": s["n_split_tensors"],
                    "swap_MB": s["d2h_bytes"] >> 20, "replays": s["n_replay"]}
        print(key, json.dumps(out[key]), flush=True)
        del S
        torch.cuda.empty_cache()
