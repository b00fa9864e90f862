"""Max trainable batch x hidden under the device's HBM (BASELINE metric part 2, config 5):
for each hidden size h (heads = h/64, FFN = 4h, 24 layers, s512) find the largest batch
that (a) fits unsplit ("Base") and (b) the TSPLIT planner fits into the free HBM,
then run 2 steps of (b) on the GPU (zero-initialised weights: op times and memory do not
depend on the values) and report samples/s.

    python tools/max_scale.py [--hidden 1024,2560] [--batches 8,16,32,64,128,256]
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--hidden", default="1024,1536,2048,2560")
    ap.add_argument("--batches", default="8,16,32,64,128,256")
    ap.add_argument("--reserve-gb", type=float, default=6.0)
    ap.add_argument("--steps", type=int, default=2)
    ap.add_argument("--out", default="gpurun_out/max_scale.json")
    args = ap.parse_args()
    free, total = torch.cuda.mem_get_info()
    cap = int(free - args.reserve_gb * 2**30)
    res = {"device_free_bytes": free, "device_total_bytes": total, "capacity_bytes": cap, "rows": []}
    print(f"capacity {cap/1e9:.1f} GB of {total/1e9:.1f} GB", flush=True)
    for h in [int(x) for x in args.hidden.split(",")]:
        best_base, best_ts = None, None
        for b in [int(x) for x in args.batches.split(",")]:
            spec = graphs.bert(layers=24, hidden=h, heads=h // 64, batch=b)
            G = tsplit.Graph(spec)
            base = tsplit.Plan.default(G).stats()
            row = {"hidden": h, "batch": b, "unsplit_peak": base["peak_extent"], "static": base["static_bytes"]}
            if base["peak_extent"] <= cap:
                best_base = (b, base["peak_extent"])
            if base["static_bytes"] >= cap:
                row["feasible"] = False
                res["rows"].append(row)
                print(json.dumps(row), flush=True)
                break
            t0 = time.time()
            try:
                P = tsplit.Plan.plan(G, cap)
                st = P.stats()
                row.update(feasible=True, plan_peak=st["peak_extent"], plan_s=round(time.time() - t0, 1),
                           predicted_ms=st["predicted_s"] * 1e3, swap_bytes=st["d2h_bytes"],
                           recompute_tensors=st["n_recompute_tensors"], split_tensors=st["n_split_tensors"])
                best_ts = (b, P, G, spec)
            except tsplit.TsError as e:
                row.update(feasible=False, error=str(e)[:120])
                res["rows"].append(row)
                print(json.dumps(row), flush=True)
                break
            res["rows"].append(row)
            print(json.dumps(row), flush=True)
        entry = {"hidden": h, "max_batch_unsplit": best_base[0] if best_base else 0,
                 "max_batch_tsplit": best_ts[0] if best_ts else 0}
        if best_ts:
            b, P, G, spec = best_ts
            S = tsplit.Session(G, P, lr=0.0)
            dev = tsplit.inputs_to_device(G, gen.make_inputs(spec))
            loss = S.step(dev)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            for _ in range(args.steps):
                loss = S.step(dev)
            dt = (time.perf_counter() - t0) / args.steps
            entry.update(samples_per_s=b / dt, ms_per_step=dt * 1e3, loss=loss,
                         scale=b * h, scale_unsplit=entry["max_batch_unsplit"] * h)
            del S
            torch.cuda.empty_cache()
        res.setdefault("summary", []).append(entry)
        print(json.dumps(entry), flush=True)
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump(res, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
