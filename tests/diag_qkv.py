"""Diagnostic (not collected): q/k/v split plans on bert_small, per tensor vs the oracle."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
from conftest import global_rel_err, rel_errs  # noqa: E402
from oracle import net  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def run(g, cfg, env):
    for k, v in env.items():
        os.environ[k] = v
    try:
        G = tsplit.Graph(g)
        P = tsplit.Plan.default(G)
        for t, c in cfg.items():
            P.set(t, *c)
        S = tsplit.Session(G, P)
        S.set_params(gen.init_params(g))
        S.step(tsplit.inputs_to_device(G, gen.make_inputs(g)))
        return S.grads()
    finally:
        for k in env:
            os.environ.pop(k, None)


for fa in (True, False):
    for batch, seq in ((8, 128), (4, 128), (8, 64)):
        g = graphs.config_graph("bert_small", fused_attention=fa, batch=batch, seq=seq)
        names = {t["name"]: t["id"] for t in g["tensors"]}
        _, og, _, _ = net.train_step(g, gen.init_params(g), gen.make_inputs(g))
        for label, cfg in (("none", {}), ("qkv p2", {names[f"l1.{x}"]: (0, 2, 1) for x in "qkv"}),
                           ("q p2", {names["l1.q"]: (0, 2, 1)})):
            for env in ({}, {"TSPLIT_NO_FUSION": "1"}):
                gr = run(g, cfg, env)
                e = rel_errs(gr, og)
                w = sorted(e.items(), key=lambda kv: -kv[1])[:3]
                print(f"fa={fa} b{batch} s{seq} {label:7s} {env} worst", [(k, round(v, 4)) for k, v in w], flush=True)
