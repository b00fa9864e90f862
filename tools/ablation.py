"""Planner breakdown on the GPU (§VI.C):

* Fig. 14(a)-style: under a FIXED HBM budget (the config's budget in bytes), grow the batch and
  measure samples/s for TSPLIT, "TSPLIT w/o Split" (TS_PLAN_NO_SPLIT) and memory-centric
  recompute only (TS_PLAN_MEMORY_CENTRIC); report the largest batch each variant trains and the
  largest whose throughput stays >= x% of the base throughput (all-reside plan at the config
  batch, unbudgeted).
* Fig. 14(b)-style: bytes swapped out / recomputed by each plan.

    python tools/ablation.py [bert_large|vgg16] [out.json]
Synthetic inputs (tsinputs.gen), random-init weights; each point: measured profile, plan, 2
warm-up + 5 timed steps (CUDA events on the session's stream)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402

wl = sys.argv[1] if len(sys.argv) > 1 else "bert_large"
out = sys.argv[2] if len(sys.argv) > 2 else f"gpurun_out/ablation_{wl}.json"
if wl == "bert_large":
    base_batch, frac, batches = 32, 0.25, [32, 48, 64, 96, 128]
    mk = lambda b: graphs.bert(layers=24, batch=b, fused_attention=True)  # noqa: E731
else:
    base_batch, frac, batches = 64, 0.30, [64, 96, 128, 192, 256]
    mk = lambda b: graphs.config_graph("vgg16", batch=b)  # noqa: E731

VARIANTS = {"tsplit": {}, "no_split": {"no_split": True}, "memory_centric": {"memory_centric": True}}


def run(spec, plan, G, dev):
    stream = torch.cuda.Stream()
    S = tsplit.Session(G, plan, lr=1e-4, streams=(stream, torch.cuda.Stream(), torch.cuda.Stream()))
    S.set_params(gen.init_params(spec, seed=1))
    for _ in range(2):
        S.step(dev)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    for _ in range(5):
        S.step_async(dev)
    e1.record(stream)
    torch.cuda.synchronize()
    del S
    torch.cuda.empty_cache()
    return e0.elapsed_time(e1) / 5 / 1e3


def swapped_recomputed(spec, plan):
    sw = rc = 0
    for t in spec["tensors"]:
        if t["kind"] != "act":
            continue
        o = plan.get(t["id"])[0]
        nbytes = 1
        for d in t["shape"]:
            nbytes *= d
        nbytes *= 2 if t["dtype"] == "bf16" else 4
        sw += nbytes if o == tsplit.SWAP else 0
        rc += nbytes if o == tsplit.RECOMPUTE else 0
    return sw, rc


spec0 = mk(base_batch)
G0 = tsplit.Graph(spec0)
st0 = tsplit.Plan.default(G0).stats()
budget = st0["static_bytes"] + int(frac * (st0["peak_extent"] - st0["static_bytes"]))
dev0 = tsplit.inputs_to_device(G0, gen.make_inputs(spec0))
base_s = run(spec0, tsplit.Plan.default(G0), G0, dev0)
base_tput = base_batch / base_s
del dev0
rows = []
for b in batches:
    spec = mk(b)
    G = tsplit.Graph(spec)
    dev = tsplit.inputs_to_device(G, gen.make_inputs(spec))
    t0 = time.time()
    prof = tsplit.Profile.measure(G, dev, max_p=16)
    prof_s = time.time() - t0
    for name, kw in VARIANTS.items():
        row = {"batch": b, "variant": name}
        try:
            P = tsplit.Plan.plan(G, budget, prof, **kw)
        except tsplit.TsError as e:
            row.update(feasible=False, why=str(e)[:120])
            rows.append(row)
            print(json.dumps(row), flush=True)
            continue
        s = P.stats()
        sw, rc = swapped_recomputed(spec, P)
        sec = run(spec, P, G, dev)
        row.update(feasible=True, samples_per_s=b / sec, frac_of_base=(b / sec) / base_tput,
                   peak_extent=s["peak_extent"], split_tensors=s["n_split_tensors"], replays=s["n_replay"],
                   swapped_bytes=sw, recomputed_bytes=rc, recompute_cache_bytes=s["recompute_cache_bytes"],
                   predicted_ms=1e3 * s["predicted_s"])
        rows.append(row)
        print(json.dumps(row), flush=True)
    del dev
    torch.cuda.empty_cache()
summary = {}
for name in VARIANTS:
    ok = [r for r in rows if r["variant"] == name and r["feasible"]]
    summary[name] = {"max_batch": max((r["batch"] for r in ok), default=None)}
    for x in (0.6, 0.5):
        summary[name][f"max_batch_at_{int(100 * x)}pct_base"] = max(
            (r["batch"] for r in ok if r["frac_of_base"] >= x), default=None)
res = {"workload": wl, "budget_bytes": budget, "budget_frac_of_b%d_dynamic" % base_batch: frac,
       "base": {"batch": base_batch, "samples_per_s": base_tput, "plan": "all reside, unbudgeted"},
       "rows": rows, "summary": summary}
json.dump(res, open(out, "w"), indent=1)
print(json.dumps(summary))
