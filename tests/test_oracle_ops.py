"""Pins of oracle/ops.py against things other than itself:
central finite differences, closed forms, invariants and published test vectors."""

import numpy as np
import pytest

from oracle import net, ops
from tsinputs import gen, graphs

rng = np.random.default_rng(7)
H = 1e-6


def fd_check(f, args, idx, dy, analytic, n=6):
    """Compare <dy, df/dargs[idx]> along random directions with central differences."""
    x = args[idx]
    for _ in range(n):
        d = rng.standard_normal(x.shape)
        a1 = list(args); a1[idx] = x + H * d
        a2 = list(args); a2[idx] = x - H * d
        num = float(np.sum(dy * (f(*a1) - f(*a2)))) / (2 * H)
        ana = float(np.sum(analytic * d))
        assert abs(num - ana) <= 1e-6 * max(1.0, abs(ana)), (num, ana)


def test_linear_fd():
    x, w, b = rng.standard_normal((5, 4)), rng.standard_normal((3, 4)), rng.standard_normal(3)
    dy = rng.standard_normal((5, 3))
    dx, dw, db = ops.linear_bwd(dy, x, w)
    fd_check(ops.linear_fwd, [x, w, b], 0, dy, dx)
    fd_check(ops.linear_fwd, [x, w, b], 1, dy, dw)
    fd_check(ops.linear_fwd, [x, w, b], 2, dy, db)


def test_elementwise_fd():
    x = rng.standard_normal((4, 7))
    x[np.abs(x) < 1e-3] = 0.5  # keep away from the ReLU kink
    dy = rng.standard_normal(x.shape)
    fd_check(ops.relu_fwd, [x], 0, dy, ops.relu_bwd(dy, ops.relu_fwd(x)))
    fd_check(ops.gelu_fwd, [x], 0, dy, ops.gelu_bwd(dy, x))
    fd_check(ops.tanh_fwd, [x], 0, dy, ops.tanh_bwd(dy, ops.tanh_fwd(x)))
    fd_check(ops.softmax_fwd, [x], 0, dy, ops.softmax_bwd(dy, ops.softmax_fwd(x)))


def test_gelu_closed_forms():
    # GELU(0) = 0, GELU'(0) = 1/2, GELU(x) -> x for large x, -> 0 for very negative x
    assert ops.gelu_fwd(np.array([0.0]))[0] == 0.0
    assert abs(ops.gelu_bwd(np.array([1.0]), np.array([0.0]))[0] - 0.5) < 1e-15
    assert abs(ops.gelu_fwd(np.array([10.0]))[0] - 10.0) < 1e-12
    # GELU(1) = Phi(1) = 0.8413447460685429 (standard normal CDF)
    assert abs(ops.gelu_fwd(np.array([1.0]))[0] - 0.8413447460685429) < 1e-15


def test_layernorm_fd_and_moments():
    x = rng.standard_normal((6, 16)) * 3 + 1
    g, b = rng.standard_normal(16), rng.standard_normal(16)
    dy = rng.standard_normal(x.shape)
    dx, dg, db = ops.layernorm_bwd(dy, x, g, 1e-12)
    f = lambda x_, g_, b_: ops.layernorm_fwd(x_, g_, b_, 1e-12)
    fd_check(f, [x, g, b], 0, dy, dx)
    fd_check(f, [x, g, b], 1, dy, dg)
    fd_check(f, [x, g, b], 2, dy, db)
    y = ops.layernorm_fwd(x, np.ones(16), np.zeros(16), 0.0)
    assert np.allclose(y.mean(-1), 0, atol=1e-13) and np.allclose(y.var(-1), 1, atol=1e-12)


def test_softmax_rows_sum_to_one():
    y = ops.softmax_fwd(rng.standard_normal((3, 2, 5, 9)) * 20)
    assert np.allclose(y.sum(-1), 1.0, atol=1e-14) and (y >= 0).all()


def test_attention_fd_and_loops():
    heads, seq, d, nb = 2, 3, 4, 2
    q = rng.standard_normal((nb * seq, heads * d))
    k = rng.standard_normal((nb * seq, heads * d))
    v = rng.standard_normal((nb * seq, heads * d))
    alpha = 0.5
    s = ops.attn_qk_fwd(q, k, heads, seq, alpha)
    # direct loops (textbook definition of per-head scores)
    for bb in range(nb):
        for a in range(heads):
            for i in range(seq):
                for j in range(seq):
                    ref = alpha * sum(q[bb * seq + i, a * d + e] * k[bb * seq + j, a * d + e] for e in range(d))
                    assert abs(s[bb, a, i, j] - ref) < 1e-12
    ds = rng.standard_normal(s.shape)
    dq, dk = ops.attn_qk_bwd(ds, q, k, heads, seq, alpha)
    f = lambda q_, k_: ops.attn_qk_fwd(q_, k_, heads, seq, alpha)
    fd_check(f, [q, k], 0, ds, dq)
    fd_check(f, [q, k], 1, ds, dk)
    p = ops.softmax_fwd(s)
    c = ops.attn_pv_fwd(p, v, heads, seq)
    for bb in range(nb):
        for a in range(heads):
            for i in range(seq):
                for e in range(d):
                    ref = sum(p[bb, a, i, j] * v[bb * seq + j, a * d + e] for j in range(seq))
                    assert abs(c[bb * seq + i, a * d + e] - ref) < 1e-12
    dc = rng.standard_normal(c.shape)
    dp, dv = ops.attn_pv_bwd(dc, p, v, heads, seq)
    g = lambda p_, v_: ops.attn_pv_fwd(p_, v_, heads, seq)
    fd_check(g, [p, v], 0, dc, dp)
    fd_check(g, [p, v], 1, dc, dv)


def test_embed_and_cls():
    V, S, hd, nb = 11, 4, 3, 2
    ids = rng.integers(0, V, nb * S)
    tt = rng.integers(0, 2, nb * S)
    ww, wp, wt = rng.standard_normal((V, hd)), rng.standard_normal((S, hd)), rng.standard_normal((2, hd))
    y = ops.embed_fwd(ids, tt, ww, wp, wt, S, 0)
    for r in range(nb * S):
        assert np.allclose(y[r], ww[ids[r]] + wp[r % S] + wt[tt[r]])
    dy = rng.standard_normal(y.shape)
    dw, dp, dt = ops.embed_bwd(dy, ids, tt, S, 0, [ww.shape, wp.shape, wt.shape])
    f = lambda a, b, c: ops.embed_fwd(ids, tt, a, b, c, S, 0)
    fd_check(f, [ww, wp, wt], 0, dy, dw)
    fd_check(f, [ww, wp, wt], 1, dy, dp)
    fd_check(f, [ww, wp, wt], 2, dy, dt)
    # a block starting at sample 1 sees positions 0..S-1 again
    assert np.allclose(ops.embed_fwd(ids[S:], tt[S:], ww, wp, wt, S, S), y[S:])
    x = rng.standard_normal((nb * S, hd))
    assert np.allclose(ops.cls_fwd(x, S), x[[0, S]])
    dyc = rng.standard_normal((nb, hd))
    fd_check(lambda x_: ops.cls_fwd(x_, S), [x], 0, dyc, ops.cls_bwd(dyc, S, nb * S))


def test_xent_closed_forms_and_fd():
    # uniform logits: CE = log C for every sample
    z = np.zeros((4, 10))
    assert abs(ops.xent_fwd(z, np.arange(4), 4) - np.log(10)) < 1e-14
    # global-batch normalisation (R14): two halves sum to the whole
    z = rng.standard_normal((6, 5)); lab = rng.integers(0, 5, 6)
    whole = ops.xent_fwd(z, lab, 6)
    assert abs(ops.xent_fwd(z[:3], lab[:3], 6) + ops.xent_fwd(z[3:], lab[3:], 6) - whole) < 1e-14
    d = ops.xent_bwd(z, lab, 6)
    fd_check(lambda z_: np.array([ops.xent_fwd(z_, lab, 6)]), [z], 0, np.ones(1), d)


def test_philox_known_answers():
    """Random123 Philox4x32-10 known-answer vectors (kat_vectors)."""
    u = lambda *v: tuple(np.array([x], np.uint64) for x in v)
    out = ops.philox4x32_10(u(0, 0, 0, 0), 0, 0)
    assert [int(o[0]) for o in out] == [0x6627e8d5, 0xe169c58d, 0xbc57ac4c, 0x9b00dbd8]
    out = ops.philox4x32_10(u(0xffffffff, 0xffffffff, 0xffffffff, 0xffffffff), 0xffffffff, 0xffffffff)
    assert [int(o[0]) for o in out] == [0x408f276d, 0x41c83b0e, 0xa20bc7c6, 0x6d5451fd]
    out = ops.philox4x32_10(u(0x243f6a88, 0x85a308d3, 0x13198a2e, 0x03707344), 0xa4093822, 0x299f31d0)
    assert [int(o[0]) for o in out] == [0xd16cfe09, 0x94fdcceb, 0x5001e420, 0x24126ea1]


def test_dropout_draws_are_the_philox_halves():
    """D-RNG: elements 8c .. 8c+7 take the low / high 16-bit halves of the four words of
    Philox call c in order (checked against the pinned philox4x32_10 on counters 0 and 5)."""
    u = lambda *v: tuple(np.array([x], np.uint64) for x in v)
    for c in (0, 5):
        w = [int(o[0]) for o in ops.philox4x32_10(u(c, 0, 3, 0), 42, ops.PHILOX_KEY1)]
        halves = [h for x in w for h in (x & 0xFFFF, x >> 16)]
        got = ops.philox_word(np.arange(8 * c, 8 * c + 8, dtype=np.uint64), 42, 3)
        assert [int(v) for v in got] == halves
        keep = ops.dropout_keep((8,), 8 * c, 0.3, 42, 3)
        assert list(keep) == [h >= int(0.3 * 65536) for h in halves]


def test_dropout_rate_and_split_invariance():
    keep = ops.dropout_keep((1 << 16,), 0, 0.1, 42)
    assert abs(keep.mean() - 0.9) < 0.01
    # the mask of a block equals the corresponding slice of the whole mask (R15)
    assert (ops.dropout_keep((100,), 300, 0.1, 42) == keep[300:400]).all()
    x = rng.standard_normal(50)
    y = ops.dropout_fwd(x, 0.25, 3, 0)
    k = ops.dropout_keep((50,), 0, 0.25, 3)
    assert np.allclose(y[k], x[k] / 0.75) and (y[~k] == 0).all()


def test_round_bf16_pins():
    """ops.round_bf16 (the bf16 storage reading, SURVEY R20 / DESIGN D-TOL): exact
    ties-to-even cases worked by hand, and agreement with torch's own fp32 -> bf16
    conversion (a library routine) on random and edge values."""
    from oracle import ops as O
    # spacing of bf16 at 1.0 is 2^-7: 1 + 2^-8 ties -> 1 (even), 1 + 3*2^-8 ties -> 1 + 2^-6 (even)
    assert O.round_bf16(np.array([1 + 2.0 ** -8]))[0] == 1.0
    assert O.round_bf16(np.array([1 + 3 * 2.0 ** -8]))[0] == 1 + 2.0 ** -6
    assert O.round_bf16(np.array([1 + 2.0 ** -8 + 2.0 ** -20]))[0] == 1 + 2.0 ** -7
    assert O.round_bf16(np.array([-3.0]))[0] == -3.0
    torch = pytest.importorskip("torch")
    r = np.random.default_rng(0)
    x = np.concatenate([r.standard_normal(100000) * 10.0 ** r.integers(-30, 30, 100000),
                        [0.0, -0.0, 1e-40, -1e-39, 3.3895e38]])
    ref = torch.from_numpy(x.astype(np.float32)).to(torch.bfloat16).to(torch.float64).numpy()
    assert np.array_equal(O.round_bf16(x), ref)


def test_bf16_storage_reading():
    """train_step(storage="bf16") rounds exactly the stored values: every activation it
    keeps is bf16-representable, parameter gradients stay unrounded, and the result is
    close to (but not equal to) the fp64 definition."""
    from oracle import ops as O
    g = graphs.config_graph("bert_tiny", layers=1)
    P, I = gen.init_params(g), gen.make_inputs(g)
    l0, g0, _, _ = net.train_step(g, P, I)
    l1, g1, val, grad = net.train_step(g, P, I, storage="bf16")
    acts = [t["id"] for t in g["tensors"] if t["kind"] == "act" and t["dtype"] == "bf16"]
    for tid in acts:
        assert np.array_equal(O.round_bf16(val[tid]), val[tid])
        if tid in grad:
            assert np.array_equal(O.round_bf16(grad[tid]), grad[tid])
    assert any(not np.array_equal(O.round_bf16(v), v) for v in g1.values())
    assert abs(l1 - l0) <= 1e-2 * abs(l0)
    num = sum(float(np.sum((g1[k] - g0[k]) ** 2)) for k in g0)
    den = sum(float(np.sum(g0[k] ** 2)) for k in g0)
    assert 0 < (num / den) ** 0.5 <= 5e-2
