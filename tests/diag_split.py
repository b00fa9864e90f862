"""Diagnostic (not collected): per-tensor split-vs-unsplit differences of a bf16 graph."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
from conftest import global_rel_err, rel_errs  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def run(g, budget=None, cfg=None):
    G = tsplit.Graph(g)
    P = tsplit.Plan.plan(G, budget) if budget else tsplit.Plan.default(G)
    for t, c in (cfg or {}).items():
        P.set(t, *c)
    S = tsplit.Session(G, P)
    S.set_params(gen.init_params(g))
    S.step(tsplit.inputs_to_device(G, gen.make_inputs(g)))
    return S.grads(), P


g = graphs.config_graph("bert_small", fused_attention=True)
g0, P0 = run(g)
g0b, _ = run(g)
print("all-reside run-to-run:", global_rel_err(g0b, g0))
base = P0.stats()
budget = base["static_bytes"] + (base["peak_extent"] - base["static_bytes"]) * 4 // 10
g1, P1 = run(g, budget)
names = {t["id"]: t["name"] for t in g["tensors"]}
print("plan:", {names[t]: c for t, c in P1.cfg_dict().items() if tuple(c[:2]) != (0, 1)})
e = rel_errs(g1, g0)
print("split vs unsplit global", global_rel_err(g1, g0), sorted(e.items(), key=lambda kv: -kv[1])[:8])
for t, c in P1.cfg_dict().items():
    if tuple(c[:2]) == (0, 1):
        continue
    gi, _ = run(g, cfg={t: tuple(c[:3])})
    print(names[t], c, "alone:", round(global_rel_err(gi, g0), 6))
