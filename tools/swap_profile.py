"""Swap traffic of a budgeted step on the GPU: achieved D2H / H2D bandwidth of every
swap-out / swap-in copy (cudaEvent pairs on the copy streams, eager profiled step) against
the measured pinned PCIe bandwidth (ts_profile_measure), the links' busy share of the
step, and how much of the copy time the compute stream hides (graph-mode step time vs the
compute stream's own busy time).  North_star: "swap traffic against the measured per-GPU
PCIe Gen5 H2D/D2H bandwidth".

    python tools/swap_profile.py resnet50 [budget_frac]   -> gpurun_out/swap_profile_<wl>.json
    python tools/swap_profile.py bert_large [budget_frac] [swap_layers]
      (bert: the planned 25 % plan, plus a forced variant that swaps the FFN1 outputs of the
       first `swap_layers` layers instead of the planner's choice for them)
"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def piece_bytes(spec, plan, key):
    t = spec["tensors"][key % len(spec["tensors"])]
    n = int(np.prod(t["shape"])) * {"bf16": 2, "f32": 4, "i32": 4}[t["dtype"]]
    return n // plan.get(t["id"])[1]


def measure(spec, G, plan, params, dev, steps=10):
    S = tsplit.Session(G, plan, lr=1e-4)
    S.set_params(params)
    for _ in range(3):
        S.step_async(dev)
    torch.cuda.synchronize()
    st = torch.cuda.current_stream()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(st)
    for _ in range(steps):
        S.step_async(dev)
    torch.cuda.synchronize()  # the session's own streams
    e1.record(st)
    torch.cuda.synchronize()
    step_ms = e0.elapsed_time(e1) / steps
    S.profile_items(True)
    S.step(dev)
    eager = S.item_times()
    S.profile_items(False)
    items = plan.items()
    so = [(piece_bytes(spec, plan, aux >> 16), t) for (k, _, _, aux), t in zip(items, eager) if k == "SO"]
    si = [(piece_bytes(spec, plan, aux >> 16), t) for (k, _, _, aux), t in zip(items, eager) if k == "SI"]
    busy = sum(t for (k, _, _, _), t in zip(items, eager) if k in ("F", "B", "R"))
    del S
    torch.cuda.empty_cache()

    def link(cp):
        if not cp:
            return None
        b = sum(x for x, _ in cp)
        t = sum(y for _, y in cp)
        per = [x / y / 1e6 for x, y in cp if y > 0]
        return {"copies": len(cp), "bytes": b, "copy_ms": t, "achieved_gbs": b / t / 1e6,
                "median_copy_gbs": statistics.median(per), "busy_share_of_step": t / step_ms}
    return {"ms_per_step_graph": step_ms, "compute_busy_ms_eager": busy,
            "exposed_ms": max(0.0, step_ms - busy), "d2h": link(so), "h2d": link(si)}


def main():
    wl = sys.argv[1] if len(sys.argv) > 1 else "resnet50"
    frac = float(sys.argv[2]) if len(sys.argv) > 2 else 0.25
    if wl == "resnet50":
        spec = graphs.resnet50(batch=256)
    elif wl == "vgg16":
        spec = graphs.vgg16(batch=64)
    else:
        spec = graphs.bert(layers=24, batch=32, fused_attention=True)
    G = tsplit.Graph(spec)
    base = tsplit.Plan.default(G).stats()
    budget = base["static_bytes"] + int(frac * (base["peak_extent"] - base["static_bytes"]))
    params = gen.init_params(spec)
    dev = tsplit.inputs_to_device(G, gen.make_inputs(spec))
    prof = tsplit.Profile.measure(G, dev, max_p=16)
    d2h_bw, h2d_bw = prof.pcie()
    plan = tsplit.Plan.plan(G, budget, prof)
    out = {"workload": wl, "budget_bytes": budget, "budget_frac": frac,
           "measured_pcie_gbs": {"d2h": d2h_bw / 1e9, "h2d": h2d_bw / 1e9}, "plans": {}}
    variants = [("planned", plan)]
    if wl == "vgg16" and len(sys.argv) > 3:  # C2's "conv offload": swap conv #i's output
        convs = [o for o in spec["ops"] if o["kind"] == "conv2d"]
        t = convs[int(sys.argv[3])]["outputs"][0]
        for lead, lag in ((1, 0), (4, 4), (16, 24)):
            forced = tsplit.Plan.deserialize(G, plan.serialize())
            forced.set(t, tsplit.SWAP, forced.get(t)[1], lead, 0, lag)
            if forced.stats()["peak_extent"] <= budget:
                variants.append((f"conv{sys.argv[3]}_offload_lead{lead}_lag{lag}", forced))
    if wl == "bert_large" and len(sys.argv) > 3:
        names = {t["name"]: t["id"] for t in spec["tensors"]}
        for lead, lag in ((4, 0), (8, 8), (16, 16), (32, 24)):
            forced = tsplit.Plan.deserialize(G, plan.serialize())
            for l in range(int(sys.argv[3])):
                forced.set(names[f"l{l}.ffn1"], tsplit.SWAP, 1, lead, 0, lag)
            fs = forced.stats()
            print("forced", lead, lag, fs["peak_extent"] <= budget, fs["predicted_s"] * 1e3, plan.stats()["predicted_s"] * 1e3,
                  flush=True)
            if fs["peak_extent"] <= budget:
                variants.append((f"ffn1_swapped_first_{sys.argv[3]}_lead{lead}_lag{lag}", forced))
    for name, P in variants:
        st = P.stats()
        r = measure(spec, G, P, params, dev)
        r["plan"] = {"d2h_bytes": st["d2h_bytes"], "h2d_bytes": st["h2d_bytes"], "n_swap_tensors": st["n_swap_tensors"],
                     "n_recompute_tensors": st["n_recompute_tensors"], "peak_extent": st["peak_extent"]}
        out["plans"][name] = r
        print(name, json.dumps(r), flush=True)
    os.makedirs("gpurun_out", exist_ok=True)
    json.dump(out, open(f"gpurun_out/swap_profile_{wl}.json", "w"), indent=1)


if __name__ == "__main__":
    main()
