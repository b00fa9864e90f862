"""Pins of the oracle's CNN ops and nets (configs 2-3): direct loops, finite
differences, BN moments, and plan invariance with batch-statistics BN (R13)."""

import random

import numpy as np
import pytest

from conftest import rel_errs
from oracle import brute, execplan, net, ops
from test_oracle_ops import fd_check
from tsinputs import gen, graphs

rng = np.random.default_rng(11)


@pytest.mark.parametrize("stride,pad,R", [(1, 1, 3), (2, 1, 3), (1, 0, 1), (2, 0, 1), (2, 3, 7)])
def test_conv2d_direct_loop_and_fd(stride, pad, R):
    N, H, C, K = 2, 9, 3, 4
    x = rng.standard_normal((N, H, H, C))
    w = rng.standard_normal((K, R, R, C))
    b = rng.standard_normal(K)
    y = ops.conv2d_fwd(x, w, b, stride, pad)
    P = (H + 2 * pad - R) // stride + 1
    assert y.shape == (N, P, P, K)
    for n in range(N):
        for p in range(P):
            for q in range(P):
                for k in range(K):
                    acc = b[k]
                    for r in range(R):
                        for s in range(R):
                            h, ww = p * stride + r - pad, q * stride + s - pad
                            if 0 <= h < H and 0 <= ww < H:
                                acc += float(np.dot(x[n, h, ww], w[k, r, s]))
                    assert abs(y[n, p, q, k] - acc) < 1e-12
    dy = rng.standard_normal(y.shape)
    dx, dw, db = ops.conv2d_bwd(dy, x, w, stride, pad)
    f = lambda x_, w_, b_: ops.conv2d_fwd(x_, w_, b_, stride, pad)
    fd_check(f, [x, w, b], 0, dy, dx)
    fd_check(f, [x, w, b], 1, dy, dw)
    fd_check(f, [x, w, b], 2, dy, db)


def test_batchnorm_fd_and_moments():
    x = rng.standard_normal((3, 4, 4, 5)) * 2 + 0.5
    g, b = rng.standard_normal(5), rng.standard_normal(5)
    y = ops.batchnorm_fwd(x, np.ones(5), np.zeros(5), 0.0)
    assert np.allclose(y.mean(axis=(0, 1, 2)), 0, atol=1e-13) and np.allclose(y.var(axis=(0, 1, 2)), 1, atol=1e-12)
    dy = rng.standard_normal(x.shape)
    dx, dg, db = ops.batchnorm_bwd(dy, x, g, 1e-5)
    f = lambda x_, g_, b_: ops.batchnorm_fwd(x_, g_, b_, 1e-5)
    fd_check(f, [x, g, b], 0, dy, dx)
    fd_check(f, [x, g, b], 1, dy, dg)
    fd_check(f, [x, g, b], 2, dy, db)
    # split form (full-batch statistics, per-block normalisation) equals the whole
    mu, var = ops.batchnorm_stats(x)
    assert np.allclose(ops.batchnorm_fwd_with(x[:1], g, b, mu, var, 1e-5), ops.batchnorm_fwd(x, g, b, 1e-5)[:1])
    s1, s2, dgs, dbs = ops.batchnorm_bwd_sums(dy, x, g, mu, var, 1e-5)
    m = 3 * 4 * 4
    assert np.allclose(ops.batchnorm_bwd_with(dy[2:], x[2:], g, mu, var, s1, s2, m, 1e-5), dx[2:])
    assert np.allclose(dgs, dg) and np.allclose(dbs, db)


@pytest.mark.parametrize("k,stride,pad", [(2, 2, 0), (3, 2, 1)])
def test_pooling(k, stride, pad):
    x = rng.permutation(2 * 6 * 6 * 3).reshape(2, 6, 6, 3).astype(float)  # distinct values: no ties
    y = ops.maxpool_fwd(x, k, stride, pad)
    P = y.shape[1]
    for n in range(2):
        for p in range(P):
            for q in range(P):
                for c in range(3):
                    vals = [x[n, h, w, c] for h in range(p * stride - pad, p * stride - pad + k)
                            for w in range(q * stride - pad, q * stride - pad + k) if 0 <= h < 6 and 0 <= w < 6]
                    assert y[n, p, q, c] == max(vals)
    dy = rng.standard_normal(y.shape)
    fd_check(lambda x_: ops.maxpool_fwd(x_, k, stride, pad), [x], 0, dy, ops.maxpool_bwd(dy, x, k, stride, pad))
    # ties: the gradient goes to the first maximum in window order (R16)
    z = np.zeros((1, 2, 2, 1))
    g = ops.maxpool_bwd(np.ones((1, 1, 1, 1)), z, 2, 2, 0)
    assert g[0, 0, 0, 0] == 1 and g.sum() == 1
    a = rng.standard_normal((2, 3, 3, 4))
    dya = rng.standard_normal((2, 4))
    fd_check(ops.avgpool_fwd, [a], 0, dya, ops.avgpool_bwd(dya, a.shape))


@pytest.mark.parametrize("gname", ["vgg_tiny", "resnet_tiny"])
def test_cnn_whole_net_fd_and_plans(gname):
    g = graphs.config_graph(gname, dtype="f32")
    P, I = gen.init_params(g), gen.make_inputs(g)
    loss, pg, _, _ = net.train_step(g, P, I)
    r = np.random.default_rng(0)
    names = [t["name"] for t in g["tensors"] if t["kind"] == "param"][:: max(1, len(pg) // 5)]
    for name in names:
        d = r.standard_normal(P[name].shape)
        h = 1e-6
        p1 = dict(P); p1[name] = P[name].astype(np.float64) + h * d
        p2 = dict(P); p2[name] = P[name].astype(np.float64) - h * d
        num = (net.train_step(g, p1, I)[0] - net.train_step(g, p2, I)[0]) / (2 * h)
        ana = float(np.sum(pg[name] * d))
        assert abs(num - ana) <= 1e-6 * max(abs(ana), 1e-3), (name, num, ana)
    rr = random.Random(5)
    for trial in range(3):
        cfg = {t: (rr.choice([0, 1, 2]), rr.choice([1, 2, 4]), 1) for t in brute.act_tensors(g)}
        full = {t["id"]: (0, 1, 1) for t in g["tensors"]}
        full.update(cfg)
        l2, pg2 = execplan.execute(g, full, P, I)
        assert abs(l2 - loss) <= 1e-12 * abs(loss)
        assert max(rel_errs(pg2, pg).values()) <= 1e-12
