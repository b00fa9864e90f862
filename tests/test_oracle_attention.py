"""Oracle pins for the fused attention op: finite differences of
attention_fwd in Q, K, V (with a fixed dropout mask), the row log-sum-exp against
scipy's logsumexp (a library routine), a direct per-(sample, head) loop, the fused
BERT graph computing the same loss and gradients as the unfused one (same seeds and
Philox counters), and plan invariance (T1) of the fused graph under random
split/swap/recompute plans — including plans that regenerate only one of its two
outputs by replay."""

import random

import numpy as np
import pytest
from scipy.special import logsumexp

from conftest import rel_errs
from oracle import brute, execplan, net
from oracle import ops as O
from tsinputs import gen, graphs

rng = np.random.default_rng(7)
H = 1e-6


def _qkv(nb=2, seq=5, heads=2, d=3):
    return [rng.standard_normal((nb * seq, heads * d)) for _ in range(3)]


@pytest.mark.parametrize("p", [0.0, 0.3])
def test_attention_fd(p):
    seq, heads = 5, 2
    q, k, v = _qkv(seq=seq, heads=heads)
    alpha = 0.7
    dc = rng.standard_normal(q.shape)
    dq, dk, dv = O.attention_bwd(dc, q, k, v, heads, seq, alpha, p, 11, 40)
    for idx, ana in enumerate((dq, dk, dv)):
        for _ in range(4):
            d = rng.standard_normal(q.shape)
            a1 = [q, k, v]; a1[idx] = a1[idx] + H * d
            a2 = [q, k, v]; a2[idx] = a2[idx] - H * d
            f1 = O.attention_fwd(*a1, heads, seq, alpha, p, 11, 40)[0]
            f2 = O.attention_fwd(*a2, heads, seq, alpha, p, 11, 40)[0]
            num = float(np.sum(dc * (f1 - f2))) / (2 * H)
            assert abs(num - float(np.sum(ana * d))) <= 1e-6 * max(1.0, abs(num))


def test_attention_loops_and_lse():
    nb, seq, heads, d = 2, 4, 3, 2
    q, k, v = _qkv(nb, seq, heads, d)
    alpha, p, seed, elem0 = 0.5, 0.25, 3, 96
    c, lse, mw = O.attention_fwd(q, k, v, heads, seq, alpha, p, seed, elem0)
    keep = O.dropout_keep((nb, heads, seq, seq), elem0, p, seed)
    # the stored keep bits: key j of a row at bit j % 32 of word j // 32
    bits = (mw.view(np.uint32)[..., :, None] >> np.arange(32, dtype=np.uint32)) & 1
    assert np.array_equal(bits.reshape(nb, heads, seq, -1)[..., :seq].astype(bool), keep)
    for b in range(nb):
        for a in range(heads):
            cols = slice(a * d, (a + 1) * d)
            qh, kh, vh = (x[b * seq:(b + 1) * seq, cols] for x in (q, k, v))
            s = alpha * qh @ kh.T
            assert np.allclose(lse[b, a], logsumexp(s, axis=1), rtol=1e-14, atol=1e-14)
            for i in range(seq):
                pr = np.exp(s[i] - logsumexp(s[i]))
                ref = sum(pr[j] * keep[b, a, i, j] / (1 - p) * vh[j] for j in range(seq))
                assert np.allclose(c[b * seq + i, cols], ref, rtol=1e-12, atol=1e-12)


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_fused_graph_equals_unfused(dtype):
    gu = graphs.config_graph("bert_tiny", dtype=dtype)
    gf = graphs.config_graph("bert_tiny", dtype=dtype, fused_attention=True)
    P, I = gen.init_params(gu), gen.make_inputs(gu)
    assert set(P) == set(gen.init_params(gf))
    lu, pu, _, _ = net.train_step(gu, P, I)
    lf, pf, vals, _ = net.train_step(gf, P, I)
    assert abs(lu - lf) <= 1e-12 * abs(lu)
    assert max(rel_errs(pf, pu).values()) <= 1e-12
    lse_ids = [t["id"] for t in gf["tensors"] if t["name"].endswith(".lse")]
    assert lse_ids and all(vals[t].dtype == np.float64 for t in lse_ids)
    mask_ids = [t["id"] for t in gf["tensors"] if t["name"].endswith(".dmask")]
    # keep fraction of the attention dropout (p = 0.1) over all layers' bits
    ones = sum(int(np.unpackbits(vals[t].view(np.uint8)).sum()) for t in mask_ids)
    total = sum(vals[t].size * 32 for t in mask_ids)
    assert abs(ones / total - 0.9) < 0.01


@pytest.mark.parametrize("seed", range(4))
def test_fused_graph_plan_invariance(seed):
    g = graphs.config_graph("bert_tiny", dtype="f32", fused_attention=True)
    P, I = gen.init_params(g), gen.make_inputs(g)
    loss, pg, _, _ = net.train_step(g, P, I)
    r = random.Random(seed)
    cfg = {t["id"]: (0, 1, 1) for t in g["tensors"]}
    for t in brute.act_tensors(g):
        cfg[t] = (r.choice([0, 1, 2]), r.choice([1, 2, 4]), 1)
    # one attention op: ctx recomputed, lse resident (and the reverse on the next layer)
    names = {t["name"]: t["id"] for t in g["tensors"]}
    cfg[names["l0.ctx"]], cfg[names["l0.lse"]] = (2, 2, 1), (0, 1, 1)
    cfg[names["l1.ctx"]], cfg[names["l1.lse"]] = (0, 1, 1), (2, 2, 1)
    l2, pg2 = execplan.execute(g, cfg, P, I)
    assert abs(l2 - loss) <= 1e-12 * abs(loss)
    assert max(rel_errs(pg2, pg).values()) <= 1e-12
