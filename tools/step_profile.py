"""Per-micro-op cudaEvent breakdown of one BERT-Large step (eager, profiled) for the
budgeted plan and the all-reside plan.  Usage: python tools/step_profile.py [budget_frac] [fused]"""
import collections
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def profile(G, P, spec, params, dev):
    S = tsplit.Session(G, P, lr=1e-4)
    S.set_params(params)
    S.step(dev)
    S.profile_items(True)
    S.step(dev)
    ms = S.item_times()
    items = P.items()
    agg = collections.Counter()
    cnt = collections.Counter()
    for (kind, op, k, aux), t in zip(items, ms):
        if kind in ("SO", "SI"):
            continue
        key = f"{kind}:{spec['ops'][op]['kind']}"
        agg[key] += t
        cnt[key] += 1
        if spec["ops"][op]["kind"] == "linear":  # per linear role (q, k, v, proj, ffn1, ffn2, ...)
            role = f"{kind}:linear.{spec['ops'][op]['name'].split('.', 1)[-1]}"
            agg[role] += t
            cnt[role] += 1
    del S
    torch.cuda.empty_cache()
    return agg, cnt, sum(t for (kind, _, _, _), t in zip(items, ms) if kind not in ("SO", "SI"))


def main():
    frac = float(sys.argv[1]) if len(sys.argv) > 1 else 0.25
    fused = len(sys.argv) > 2 and sys.argv[2] == "fused"
    spec = graphs.bert(layers=24, batch=32, fused_attention=fused)
    G = tsplit.Graph(spec)
    base = tsplit.Plan.default(G)
    st = base.stats()
    budget = st["static_bytes"] + int(frac * (st["peak_extent"] - st["static_bytes"]))
    dev0 = tsplit.inputs_to_device(G, gen.make_inputs(spec))
    prof = tsplit.Profile.measure(G, dev0, max_p=16)
    plan = tsplit.Plan.plan(G, budget, prof)
    print("plan stats", {k: v for k, v in plan.stats().items()})
    # tensors by opt
    kinds = collections.Counter()
    for t in spec["tensors"]:
        if t["kind"] == "act":
            o, p, lead = plan.get(t["id"])
            if o or p > 1:
                kinds[(t["name"].split(".", 1)[-1], o, p)] += 1
    print(sorted(kinds.items()))
    params = gen.init_params(spec)
    dev = tsplit.inputs_to_device(G, gen.make_inputs(spec))
    out = {}
    for name, P in [("budget", plan), ("unbudgeted", base)]:
        agg, cnt, tot = profile(G, P, spec, params, dev)
        print(f"== {name}: sum of item times {tot:.2f} ms")
        for k, v in agg.most_common():
            print(f"  {k:22s} {v:8.2f} ms  n={cnt[k]}")
        out[name] = {"total_ms": tot, "by_kind": dict(agg), "count": dict(cnt)}
    json.dump(out, open("gpurun_out/step_profile.json", "w"), indent=1)


if __name__ == "__main__":
    main()
