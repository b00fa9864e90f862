"""The encoder-decoder Transformer workload (IWSLT-
shaped, synthetic) on the CUDA path: fused attention in the encoder and the cross
attention, the unfused causal self-attention (attn_qk -> causal softmax -> dropout ->
attn_pv) in the decoder, a token-level loss over the vocabulary.  fp32 random plans vs the
fp64 oracle (1e-5) and vs the unsplit GPU step (1e-6); bf16 per tensor within 2e-2 of the
plain oracle, unbudgeted and under a planned budget; runtime trace = simulator."""

import random

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from conftest import assert_bf16_parity, rel_errs  # noqa: E402
from oracle import brute, net, sim  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def _run(g, cfg=None, budget=None):
    G = tsplit.Graph(g)
    if budget is not None:
        P = tsplit.Plan.plan(G, budget)
    else:
        P = tsplit.Plan.default(G)
        for t, c in (cfg or {}).items():
            P.set(t, *c)
    S = tsplit.Session(G, P)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    S.set_params(params)
    loss = S.step(tsplit.inputs_to_device(G, inputs))
    return loss, S.grads(), S, P


@pytest.mark.parametrize("seed", range(2))
def test_transformer_fp32_random_plans(seed):
    g = graphs.config_graph("transformer_tiny", dtype="f32")
    r = random.Random(900 + seed)
    cfg = {}
    for t in brute.act_tensors(g):
        o = r.choice([0, 1, 2])
        cfg[t] = (o, r.choice([1, 2, 4]), r.choice([1, 2]), 0, r.choice([0, 3]) if o == 1 else 0)
    loss, grads, S, P = _run(g, cfg)
    assert S.trace() == [tuple(e) for e in sim.simulate(g, {**sim.default_cfg(g), **cfg}).trace]
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    ol, og, _, _ = net.train_step(g, params, inputs)
    assert abs(loss - ol) <= 1e-5 * abs(ol)
    errs = rel_errs(grads, og)
    assert max(errs.values()) <= 1e-5, sorted(errs.items(), key=lambda kv: -kv[1])[:4]
    _, g0, _, _ = _run(g)
    assert max(rel_errs(grads, g0).values()) <= 1e-6


def test_transformer_bf16_parity_and_budget():
    g = graphs.config_graph("transformer_small")
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    ol, og, _, _ = net.train_step(g, params, inputs)
    loss, grads, S, P = _run(g)
    assert abs(loss - ol) <= 2e-2 * abs(ol)
    assert_bf16_parity(grads, og)
    base = P.stats()
    budget = base["static_bytes"] + (base["peak_extent"] - base["static_bytes"]) // 3
    l2, g2, S2, P2 = _run(g, budget=budget)
    st = P2.stats()
    assert st["peak_extent"] <= budget and st["n_swap_tensors"] + st["n_recompute_tensors"] > 0
    assert S2.trace() == P2.trace()
    assert_bf16_parity(g2, og)
