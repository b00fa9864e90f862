"""Max trainable scale sweep (BASELINE metric part 2, config C5; hidden grid
{1024, 1536, 2048, 2560, 3072, 4096} x batch, 24 layers, seq 512, heads = h/64, FFN = 4h).

  plan  (CPU, no GPU needed): for each hidden size, double the batch from 8 until the planner
        (Alg. 2) no longer fits the capacity; record the unsplit peak, the plan's peak / swap /
        recompute / split counts and planning time, and serialize the largest feasible plan.
        python tools/scale_sweep.py plan --capacity-bytes N [--hidden ...] [--max-batch 8192]
  run   (GPU): time 2 steps of each saved plan (zero-initialised weights; op times and memory do
        not depend on the values).   python tools/scale_sweep.py run
Output: gpurun_out/scale_sweep.json (+ .blobs/ plan blobs).
"""
import argparse
import base64
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402

OUT = "gpurun_out/scale_sweep.json"


def spec_of(h, b):
    return graphs.bert(layers=24, hidden=h, heads=h // 64, batch=b, fused_attention=True)


def plan_phase(args):
    res = {"capacity_bytes": args.capacity_bytes, "rows": [], "summary": []}
    for h in [int(x) for x in args.hidden.split(",")]:
        best_base, best = 0, None
        b = 8
        while b <= args.max_batch:
            spec = spec_of(h, b)
            G = tsplit.Graph(spec)
            base = tsplit.Plan.default(G).stats()
            row = {"hidden": h, "batch": b, "unsplit_peak": base["peak_extent"], "static": base["static_bytes"]}
            if base["peak_extent"] <= args.capacity_bytes:
                best_base = b
            if base["static_bytes"] >= args.capacity_bytes:
                row["feasible"] = False
                res["rows"].append(row)
                print(json.dumps(row), flush=True)
                break
            t0 = time.time()
            try:
                P = tsplit.Plan.plan(G, args.capacity_bytes)
                st = P.stats()
                row.update(feasible=True, plan_peak=st["peak_extent"], plan_s=round(time.time() - t0, 1),
                           predicted_ms=st["predicted_s"] * 1e3, swap_bytes=st["d2h_bytes"],
                           recompute_tensors=st["n_recompute_tensors"], split_tensors=st["n_split_tensors"])
                best = (b, base64.b64encode(P.serialize()).decode())
            except tsplit.TsError as e:
                row.update(feasible=False, error=str(e)[:160], plan_s=round(time.time() - t0, 1))
                res["rows"].append(row)
                print(json.dumps(row), flush=True)
                break
            res["rows"].append(row)
            print(json.dumps(row), flush=True)
            b *= 2
        res["summary"].append({"hidden": h, "max_batch_unsplit": best_base, "max_batch_tsplit": best[0] if best else 0,
                               "scale_unsplit": best_base * h, "scale_tsplit": (best[0] if best else 0) * h,
                               "plan_blob": best[1] if best else None,
                               "batch_cap_reached": bool(best and best[0] * 2 > args.max_batch)})
        json.dump(res, open(OUT, "w"), indent=1)


def run_phase(args):
    """Time the largest plan per hidden size whose pinned host pool (the plan's swapped
    bytes) fits the box's host memory cap; plan-feasible batches beyond it are reported as
    HBM-feasible only."""
    import torch
    res = json.load(open(args.plans or OUT))
    free, total = torch.cuda.mem_get_info()
    res["device_free_bytes"] = free
    res["host_cap_bytes"] = args.host_cap_bytes
    for s in res["summary"]:
        h = s["hidden"]
        rows = [r for r in res["rows"] if r["hidden"] == h and r.get("feasible")]
        ok = [r for r in rows if r.get("swap_bytes", 0) <= args.host_cap_bytes]
        if not ok:
            continue
        b = max(r["batch"] for r in ok)
        s["max_batch_tsplit_host_limited"] = b
        spec = spec_of(h, b)
        G = tsplit.Graph(spec)
        if b == s["max_batch_tsplit"] and s.get("plan_blob"):
            P = tsplit.Plan.deserialize(G, base64.b64decode(s["plan_blob"]))
        else:
            P = tsplit.Plan.plan(G, res["capacity_bytes"])
        S = tsplit.Session(G, P, lr=0.0, slab_bytes=res["capacity_bytes"])
        dev = tsplit.inputs_to_device(G, gen.make_inputs(spec))
        loss = S.step(dev)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(args.steps):
            loss = S.step(dev)
        dt = (time.perf_counter() - t0) / args.steps
        s.update(timed_batch=b, samples_per_s=b / dt, ms_per_step=dt * 1e3, loss=loss,
                 host_pool_bytes=S.host_pool()[0], timed_scale=b * h)
        print(json.dumps({k: v for k, v in s.items() if k != "plan_blob"}), flush=True)
        del S
        torch.cuda.empty_cache()
        json.dump(res, open(OUT, "w"), indent=1)


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("phase", choices=["plan", "run"])
    ap.add_argument("--hidden", default="1024,1536,2048,2560,3072,4096")
    ap.add_argument("--capacity-bytes", type=int, default=184404344832)
    ap.add_argument("--max-batch", type=int, default=8192)
    ap.add_argument("--steps", type=int, default=2)
    ap.add_argument("--plans", default=None, help="plan-phase output to run (default: " + OUT + ")")
    ap.add_argument("--host-cap-bytes", type=int, default=100 * 2 ** 30,
                    help="largest pinned swap pool to run (the GPU box has ~196 GB of host RAM)")
    a = ap.parse_args()
    os.makedirs("gpurun_out", exist_ok=True)
    plan_phase(a) if a.phase == "plan" else run_phase(a)
