"""Planner cost-model check: for each workload, the predicted step time of the all-reside
plan and of the budgeted plans (measured and analytic profile) against the measured
CUDA-graph step time.   python tools/predict_check.py [workload ...]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen  # noqa: E402


def step_ms(G, P, spec, params, dev, n=5):
    S = tsplit.Session(G, P, lr=1e-4)
    S.set_params(params)
    for _ in range(3):
        S.step_async(dev)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(n):
        S.step_async(dev)
    torch.cuda.synchronize()
    e1.record()
    torch.cuda.synchronize()
    del S
    torch.cuda.empty_cache()
    return e0.elapsed_time(e1) / n


out = {}
for wl in sys.argv[1:] or ["bert_large", "vgg16", "resnet50"]:
    W = bench.WORKLOADS[wl]
    spec = bench.workload_graph(wl)
    G = tsplit.Graph(spec)
    base = tsplit.Plan.default(G)
    st = base.stats()
    budget = st["static_bytes"] + int(W["frac"] * (st["peak_extent"] - st["static_bytes"]))
    params, dev = gen.init_params(spec), tsplit.inputs_to_device(G, gen.make_inputs(spec))
    prof = tsplit.Profile.measure(G, dev, max_p=16)
    rows = {}
    for name, P, pr in (("all_reside", base, None), ("planned_measured", tsplit.Plan.plan(G, budget, prof), prof),
                        ("planned_analytic", tsplit.Plan.plan(G, budget), None)):
        rows[name] = {"predicted_ms": P.stats()["predicted_s"] * 1e3, "measured_ms": step_ms(G, P, spec, params, dev)}
    out[wl] = rows
    print(wl, json.dumps(rows), flush=True)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/predict_check.json", "w"), indent=1)
