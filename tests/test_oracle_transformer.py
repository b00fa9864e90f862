"""Oracle pins for the encoder-decoder Transformer workload (PAPER.md
P:L306 "the IWSLT2016 dataset for Transformer"): the causal softmax against its
definition written per row, whole-net finite differences of a tiny encoder-decoder, and
T1 (any split / swap / recompute plan gives the unsplit gradients) on it."""

import random

import numpy as np
import pytest

from conftest import rel_errs
from oracle import brute, execplan, net
from oracle import ops as O
from tsinputs import gen, graphs


def test_causal_softmax_is_the_prefix_softmax():
    r = np.random.default_rng(3)
    x = r.standard_normal((2, 3, 7, 7)) * 3
    y = O.softmax_fwd(x, causal=True)
    for b in range(2):
        for a in range(3):
            for i in range(7):
                row = x[b, a, i, :i + 1]
                ref = np.exp(row - row.max()) / np.exp(row - row.max()).sum()
                assert np.allclose(y[b, a, i, :i + 1], ref, rtol=1e-14, atol=1e-15)
                assert np.all(y[b, a, i, i + 1:] == 0.0)
    # the backward formula needs no mask: y = 0 where masked gives dx = 0 there, and it is
    # the VJP of the masked map (finite differences)
    dy = r.standard_normal(x.shape)
    dx = O.softmax_bwd(dy, y)
    assert np.all(dx[..., np.triu(np.ones((7, 7), bool), 1)] == 0.0)
    d = r.standard_normal(x.shape)
    h = 1e-6
    num = (np.sum(dy * O.softmax_fwd(x + h * d, causal=True)) - np.sum(dy * O.softmax_fwd(x - h * d, causal=True))) / (2 * h)
    assert abs(num - np.sum(dx * d)) <= 1e-7 * max(1.0, abs(num))


def _tiny():
    return graphs.config_graph("transformer_tiny", dtype="f32", hidden=32, heads=2, ffn=64, seq=8, batch=2,
                               vocab=40)


def test_transformer_whole_net_fd():
    g = _tiny()
    P, I = gen.init_params(g), gen.make_inputs(g)
    loss, pg, _, _ = net.train_step(g, P, I)
    r = np.random.default_rng(0)
    for name in ["src.word", "tgt.pos", "e0.q.w", "e0.ln2.g", "d0.self.k.w", "d0.cross.v.w", "d0.cross.q.b",
                 "d0.ffn1.b", "out.w"]:
        d = r.standard_normal(P[name].shape)
        h = 1e-6
        p1 = dict(P); p1[name] = P[name].astype(np.float64) + h * d
        p2 = dict(P); p2[name] = P[name].astype(np.float64) - h * d
        num = (net.train_step(g, p1, I)[0] - net.train_step(g, p2, I)[0]) / (2 * h)
        ana = float(np.sum(pg[name] * d))
        assert abs(num - ana) <= 1e-6 * max(abs(ana), 1e-2), (name, num, ana)  # (loss ~ 60: FD noise ~ 6e-9)


@pytest.mark.parametrize("seed", range(3))
def test_t1_transformer_plans(seed):
    g = graphs.config_graph("transformer_tiny", dtype="f32", hidden=32, heads=2, ffn=64, seq=32, batch=4, vocab=40)
    P, I = gen.init_params(g), gen.make_inputs(g)
    l0, g0, _, _ = net.train_step(g, P, I)
    r = random.Random(seed)
    cfg = {t: (r.choice([0, 1, 2]), r.choice([1, 2, 4]), r.choice([1, 2])) for t in brute.act_tensors(g)}
    l1, g1 = execplan.execute(g, cfg, P, I, cache_bytes=r.choice([0, 2 ** 20]))
    assert abs(l1 - l0) <= 1e-12 * abs(l0)
    assert max(rel_errs(g1, g0).values()) <= 1e-12
