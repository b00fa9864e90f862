"""Batch-1 VGG-16 (224 x 224, bf16) under attribute (height) band splits (reading D-ATTR,
Fig. 6 / P:L125): step time of the unsplit step and of Alg. 2's plans at shrinking budgets,
with and without the split step (no_split = swap / recompute only).  wall clock around
`steps` CUDA-graph replays after warm-up (synchronised).  Output: gpurun_out/band_bench.json."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def time_plan(g, P, steps=20, warm=5):
    G = P.graph
    S = tsplit.Session(G, P)
    S.set_params(gen.init_params(g))
    x = tsplit.inputs_to_device(G, gen.make_inputs(g))
    for _ in range(warm):
        S.step(x)
    torch.cuda.synchronize()
    t0 = time.perf_counter()   # (the session runs on its own streams: wall clock around a sync)
    for _ in range(steps):
        S.step_async(x)
    torch.cuda.synchronize()
    return (time.perf_counter() - t0) * 1e3 / steps


def main():
    out = {"workload": "vgg16 batch 1, 224x224, bf16", "rows": []}
    for batch in (1, 2):
        g = graphs.config_graph("vgg16", batch=batch)
        G = tsplit.Graph(g)
        P0 = tsplit.Plan.default(G)
        st = P0.stats()
        base = time_plan(g, P0)
        out["rows"].append({"batch": batch, "budget_frac": 1.0, "plan": "unsplit", "ms": base,
                            "peak_extent": st["peak_extent"]})
        print(out["rows"][-1], flush=True)
        for frac in (0.65, 0.5, 0.45, 0.4):
            budget = st["static_bytes"] + int(frac * (st["peak_extent"] - st["static_bytes"]))
            for ns in (True, False):
                row = {"batch": batch, "budget_frac": frac, "plan": "no_split" if ns else "tsplit"}
                try:
                    P = tsplit.Plan.plan(G, budget, no_split=ns)
                except tsplit.TsError as e:
                    row["infeasible"] = str(e)[:100]
                    out["rows"].append(row)
                    print(row, flush=True)
                    continue
                cfg = P.oracle_cfg()
                s = P.stats()
                row.update(ms=time_plan(g, P), peak_extent=s["peak_extent"], predicted_ms=s["predicted_s"] * 1e3,
                           band_tensors=sum(1 for c in cfg.values() if c[1] > 1 and len(c) > 3 and c[3] == 2),
                           swap_tensors=s["n_swap_tensors"], recompute_tensors=s["n_recompute_tensors"])
                row["rel_to_unsplit"] = base / row["ms"]
                out["rows"].append(row)
                print(row, flush=True)
    os.makedirs("gpurun_out", exist_ok=True)
    json.dump(out, open("gpurun_out/band_bench.json", "w"), indent=1)


if __name__ == "__main__":
    main()
