"""Uninitialised-read guard: the dynamic pool is filled with 0x7F bytes (~3.4e38 as fp32 and
bf16) before the first step, so any piece a micro-op reads before some item wrote it — or a
gradient piece accumulated into without being zeroed first — blows the gradients up.  Random
plans of every split family (sample, channel, height / width bands) with swap and recompute,
against the fp64 oracle (fp32 graphs, 1e-5 per tensor)."""

import random

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from conftest import rel_errs  # noqa: E402
from oracle import brute, net  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def _plan(name, g, family, seed):
    r = random.Random(seed)
    if family == "sample":
        return {t: (r.choice([0, 1, 2]), r.choice([1, 2, 4]), r.choice([1, 2])) for t in brute.act_tensors(g)}
    if family == "band":
        from test_oracle_attr import _rand_attr_cfg
        return _rand_attr_cfg(g, r)
    if family == "chan4":
        from test_oracle_channel4 import rand_chan4_cfg
        return rand_chan4_cfg(g, r, min_block=4)
    from test_oracle_channel import CHAINS, channel_cfg
    return channel_cfg(g, r, CHAINS[name], prob=0.9)


CASES = [("mlp", "sample"), ("bert_tiny", "sample"), ("vgg_tiny", "sample"), ("resnet_tiny", "sample"),
         ("vgg_tiny", "band"), ("resnet_tiny", "band"), ("vgg_tiny", "chan4"), ("resnet_tiny", "chan4"),
         ("bert_tiny", "chan2"), ("mlp", "chan2")]


@pytest.mark.parametrize("case", range(len(CASES)))
@pytest.mark.parametrize("seed", range(2))
def test_poisoned_pool_step_equals_the_oracle(case, seed):
    name, family = CASES[case]
    g = graphs.config_graph(name, **({} if name == "mlp" else {"dtype": "f32"}))
    cfg = _plan(name, g, family, 900 + 10 * case + seed)
    G = tsplit.Graph(g)
    P = tsplit.Plan.default(G)
    P.set_many({t: cfg[t] for t in brute.act_tensors(g)})
    S = tsplit.Session(G, P)
    S.slab[P.stats()["static_bytes"]:].fill_(0x7F)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    S.set_params(params)
    loss = S.step(tsplit.inputs_to_device(G, inputs))
    ol, og, _, _ = net.train_step(g, params, inputs)
    assert abs(loss - ol) <= 1e-5 * abs(ol)
    errs = rel_errs(S.grads(), og)
    assert max(errs.values()) <= 1e-5, sorted(errs.items(), key=lambda kv: -kv[1])[:4]


def test_poisoned_pool_planned_bf16_bert_step():
    """A planned bf16 step (Alg. 2 at 25 % of bert_small's dynamic peak, fused attention: swaps,
    recomputes, D-LAG releases, CUDA-graph replay) gives the clean pool's gradients on a
    poisoned one."""
    from conftest import global_rel_err
    g = graphs.config_graph("bert_small", fused_attention=True)
    G = tsplit.Graph(g)
    st = tsplit.Plan.default(G).stats()
    P = tsplit.Plan.plan(G, st["static_bytes"] + (st["peak_extent"] - st["static_bytes"]) // 4)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    out = []
    for poison in (False, True):
        S = tsplit.Session(G, P)
        if poison:
            S.slab[P.stats()["static_bytes"]:].fill_(0x7F)
        S.set_params(params)
        dev = tsplit.inputs_to_device(G, inputs)
        loss = S.step(dev)
        loss = S.step(dev)   # (a graph replay: no item may depend on the previous step's pool)
        out.append((loss, S.grads()))
    assert abs(out[0][0] - out[1][0]) <= 1e-6 * abs(out[0][0])
    assert global_rel_err(out[1][1], out[0][1]) <= 1e-6
