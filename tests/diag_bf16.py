"""Diagnostic (not collected by pytest): per-tensor bf16 errors of the CUDA path against
the plain fp64 oracle and against the oracle's bf16-storage reading, for the configs the
bf16 parity tests use.  python tests/diag_bf16.py [config ...]"""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
from conftest import global_rel_err, rel_errs  # noqa: E402
from oracle import net  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402

CONFIGS = {
    "bert_small": dict(name="bert_small"),
    "bert_small_fa": dict(name="bert_small", fused_attention=True),
    "bertL_b4_l1": dict(name="bert_large", layers=1, batch=4, fused_attention=True),
    "bertL_b2_l1": dict(name="bert_large", layers=1, batch=2, fused_attention=True),
    "bertL_b4_l2": dict(name="bert_large", layers=2, batch=4, fused_attention=True),
    "vgg_small": dict(name="vgg_small"),
    "resnet_small": dict(name="resnet_small"),
}


def run(key):
    kw = dict(CONFIGS[key])
    g = graphs.config_graph(kw.pop("name"), **kw)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    t0 = time.time()
    ol, og, _, _ = net.train_step(g, params, inputs)
    _, ob, _, _ = net.train_step(g, params, inputs, storage="bf16")
    t1 = time.time()
    G = tsplit.Graph(g)
    S = tsplit.Session(G, tsplit.Plan.default(G))
    S.set_params(params)
    loss = S.step(tsplit.inputs_to_device(G, inputs))
    grads = S.grads()
    for ref_name, ref in (("plain", og), ("bf16-storage", ob)):
        e = rel_errs(grads, ref)
        worst = sorted(e.items(), key=lambda kv: -kv[1])[:4]
        print(f"{key} GPU vs {ref_name}: global {global_rel_err(grads, ref):.4f} max {worst[0][1]:.4f}",
              [(k, round(v, 4)) for k, v in worst], flush=True)
    e = rel_errs(ob, og)
    worst = sorted(e.items(), key=lambda kv: -kv[1])[:4]
    print(f"{key} bf16-storage vs plain (intrinsic): global {global_rel_err(ob, og):.4f}",
          [(k, round(v, 4)) for k, v in worst], f"oracle {t1 - t0:.1f}s loss {loss:.5f} {ol:.5f}", flush=True)


if __name__ == "__main__":
    for k in sys.argv[1:] or list(CONFIGS):
        run(k)
