"""CNN path on the GPU (configs C2 VGG-16 / C3 ResNet-50):

* the conv micro-op kernels (tcgen05 implicit GEMM for bf16, CUDA cores for fp32)
  against the fp64 oracle's im2col definition (oracle/ops.py conv2d_fwd/bwd),
  through the C ABI `ts_conv2d`, over shapes that cover ragged M/N tails,
  multi-tap K blocks (C < 64), stride-2 dgrad, 1x1 convs, the C = 3 image layer
  (scalar gather) and split-K wgrad;
* whole training steps of the tiny VGG / ResNet graphs under random split / swap /
  recompute plans against the oracle (fp32: 1e-5 per tensor; bf16: reading D-TOL-CNN —
  the bar is the precision's own distance from fp64, measured by the oracle alone),
  split vs unsplit on the GPU (fp32: 1e-6), and trace equality with the simulator.
"""

import random

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from conftest import global_rel_err, rel_errs  # noqa: E402
from oracle import brute, net, sim  # noqa: E402
from oracle import ops as O  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402

# (n, H, W, C, K, R, S, stride, pad)
GEOMS = [
    (2, 9, 11, 64, 64, 3, 3, 1, 1),     # 3x3, ragged pixel tail
    (3, 8, 8, 16, 24, 3, 3, 1, 1),      # C < 64: K blocks span taps; N tail
    (2, 15, 13, 32, 64, 3, 3, 2, 1),    # stride 2 (fractional dgrad taps)
    (2, 15, 13, 64, 128, 3, 3, 2, 1),   # stride 2, 64-channel (TMA: element strides, dgrad phases)
    (2, 17, 16, 64, 64, 7, 7, 2, 3),    # 7x7 stride 2, odd sizes (phases of unequal size)
    (2, 12, 12, 64, 256, 1, 1, 1, 0),   # 1x1
    (2, 14, 14, 64, 128, 1, 1, 2, 0),   # 1x1 stride-2 downsample
    (4, 7, 7, 256, 512, 3, 3, 1, 1),    # several 256-wide N tiles
    (8, 32, 32, 64, 64, 3, 3, 1, 1),    # long pixel reduction: split-K wgrad
    (2, 20, 20, 3, 16, 7, 7, 2, 3),     # ResNet stem-like, C = 3 (scalar gather)
    (1, 10, 10, 3, 64, 3, 3, 1, 1),     # VGG conv0-like, C = 3
]


def _rel(a, b):
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    return float(np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-30))


def _case(geom, seed=0):
    n, H, W, C, K, R, S, st, pad = geom
    P = (H + 2 * pad - R) // st + 1
    Q = (W + 2 * pad - S) // st + 1
    r = np.random.default_rng(seed)
    x = gen.snap_bf16(r.standard_normal((n, H, W, C)).astype(np.float32))
    w = gen.snap_bf16((r.standard_normal((K, R, S, C)) / np.sqrt(R * S * C)).astype(np.float32))
    b = gen.snap_bf16((0.1 * r.standard_normal(K)).astype(np.float32))
    dy = gen.snap_bf16(r.standard_normal((n, P, Q, K)).astype(np.float32))
    return x, w, b, dy, P, Q


def _dev(a, dt):
    return torch.from_numpy(np.ascontiguousarray(a, np.float32)).to("cuda").to(dt)


@pytest.mark.parametrize("geom", GEOMS, ids=lambda g: "x".join(map(str, g)))
@pytest.mark.parametrize("dtype", ["bf16", "f32", "bf16-gather"])
def test_conv_kernels_vs_oracle(geom, dtype):
    """bf16: the default dispatch (TMA-fed kernel for 64-channel layers, else the
    cp.async gather kernel); bf16-gather: the gather kernel forced (mode | 0x10)."""
    force = 0x10 if dtype == "bf16-gather" else 0
    dtype = dtype.split("-")[0]
    n, H, W, C, K, R, S, st, pad = geom
    x, w, b, dy, P, Q = _case(geom)
    tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
    X, Wt, B, DY = _dev(x, tdt), _dev(w, tdt), _dev(b, tdt), _dev(dy, tdt)
    y_ref = O.conv2d_fwd(x.astype(np.float64), w.astype(np.float64), b.astype(np.float64), st, pad)
    dx_ref, dw_ref, _ = O.conv2d_bwd(dy.astype(np.float64), x.astype(np.float64), w.astype(np.float64), st, pad)
    tc_expected = dtype == "bf16" and K % 8 == 0
    tol_act = 6e-3 if dtype == "bf16" else 1e-6   # bf16 output rounding (2^-9) dominates
    tol_w = 1e-4 if dtype == "bf16" else 1e-6     # fp32 accumulation of exact bf16 products

    Y = torch.empty((n, P, Q, K), dtype=tdt, device="cuda")
    used = tsplit.conv2d(1 | force, geom, X, Wt, None, Y, B)
    torch.cuda.synchronize()
    assert used == tc_expected
    assert _rel(Y.float().cpu().numpy(), y_ref) <= tol_act

    DW = torch.full((K, R, S, C), 0.5, dtype=torch.float32, device="cuda")
    used = tsplit.conv2d(3 | force, geom, X, Wt, DY, DW, acc=0)
    torch.cuda.synchronize()
    assert used == tc_expected
    assert _rel(DW.cpu().numpy(), dw_ref) <= tol_w
    # accumulate (merge = sum across micro-ops)
    tsplit.conv2d(3 | force, geom, X, Wt, DY, DW, acc=1)
    torch.cuda.synchronize()
    assert _rel(DW.cpu().numpy(), 2 * dw_ref) <= tol_w

    if C % 8 == 0 or dtype == "f32":
        DX = torch.empty((n, H, W, C), dtype=tdt, device="cuda")
        used = tsplit.conv2d(2 | force, geom, None, Wt, DY, DX, acc=0)
        torch.cuda.synchronize()
        assert used == (tc_expected and C % 8 == 0)
        assert _rel(DX.float().cpu().numpy(), dx_ref) <= tol_act
        tsplit.conv2d(2 | force, geom, None, Wt, DY, DX, acc=1)
        torch.cuda.synchronize()
        assert _rel(DX.float().cpu().numpy(), 2 * dx_ref) <= 2 * tol_act


def test_conv_split_micro_ops_sum_to_whole():
    """A sample split of a conv: fprop/dgrad of each block equal the rows of
    the whole-batch result bit for bit; wgrad accumulated over blocks matches the
    whole-batch wgrad to fp32 summation order."""
    geom = (4, 16, 16, 64, 128, 3, 3, 1, 1)
    n, H, W, C, K, R, S, st, pad = geom
    x, w, b, dy, P, Q = _case(geom, seed=3)
    X, Wt, B, DY = (_dev(a, torch.bfloat16) for a in (x, w, b, dy))
    Y = torch.empty((n, P, Q, K), dtype=torch.bfloat16, device="cuda")
    tsplit.conv2d(1, geom, X, Wt, None, Y, B)
    DX = torch.empty((n, H, W, C), dtype=torch.bfloat16, device="cuda")
    tsplit.conv2d(2, geom, None, Wt, DY, DX)
    DW = torch.empty((K, R, S, C), dtype=torch.float32, device="cuda")
    tsplit.conv2d(3, geom, X, Wt, DY, DW)
    Ys = torch.empty_like(Y)
    DXs = torch.empty_like(DX)
    DWs = torch.empty_like(DW)
    for k in range(2):
        sl = slice(2 * k, 2 * k + 2)
        g2 = (2,) + geom[1:]
        tsplit.conv2d(1, g2, X[sl], Wt, None, Ys[sl], B)
        tsplit.conv2d(2, g2, None, Wt, DY[sl], DXs[sl])
        tsplit.conv2d(3, g2, X[sl], Wt, DY[sl], DWs, acc=k)
    torch.cuda.synchronize()
    assert torch.equal(Y, Ys)
    assert torch.equal(DX, DXs)
    assert _rel(DWs.cpu().numpy(), DW.cpu().numpy()) <= 1e-6


def _run(g, plan_cfg=None, budget=None):
    G = tsplit.Graph(g)
    if budget is not None:
        P = tsplit.Plan.plan(G, budget)
    else:
        P = tsplit.Plan.default(G)
        for t, (o, p, lead) in (plan_cfg or {}).items():
            P.set(t, o, p, lead)
    S = tsplit.Session(G, P)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    S.set_params(params)
    loss = S.step(tsplit.inputs_to_device(G, inputs))
    return loss, S.grads(), S, P


def _oracle(g, storage=None):
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    loss, pg, _, _ = net.train_step(g, params, inputs, storage=storage)
    return loss, pg


@pytest.mark.parametrize("name", ["vgg_tiny", "resnet_tiny"])
@pytest.mark.parametrize("seed", range(2))
def test_cnn_tiny_fp32_random_plans(name, seed):
    g = graphs.config_graph(name, dtype="f32")
    r = random.Random(100 + seed)
    cfg = {t: (r.choice([0, 1, 2]), r.choice([1, 2, 4]), r.choice([1, 2])) for t in brute.act_tensors(g)}
    loss, grads, S, P = _run(g, cfg)
    ol, og = _oracle(g)
    assert abs(loss - ol) <= 1e-5 * abs(ol)
    errs = rel_errs(grads, og)
    assert max(errs.values()) <= 1e-5, sorted(errs.items(), key=lambda kv: -kv[1])[:5]
    l0, g0, _, _ = _run(g)
    e0 = rel_errs(grads, g0)
    assert max(e0.values()) <= 1e-6, sorted(e0.items(), key=lambda kv: -kv[1])[:5]
    assert S.trace() == [tuple(e) for e in sim.simulate(g, {**sim.default_cfg(g), **cfg}).trace]


@pytest.mark.parametrize("name", ["vgg_small", "resnet_small"])
def test_cnn_bf16_precision_and_budget(name):
    """bf16 CNN steps (reading D-TOL-CNN).  Any execution that stores ReLU-network
    activations in bf16 is far from fp64 here: the oracle alone, rounding only its stored
    values, is 3-17 % away on the early conv / BN gradients (tests/test_oracle_bf16_gap.py
    pins this; the mechanism is ReLU and max-pool decisions flipped by forward rounding).
    So the bar is that distance, not 2e-2: per tensor the GPU is within max(2e-2, 1.5 x)
    the bf16-storage reading's own error against the plain fp64 oracle, and the whole
    gradient within max(2e-2, 1.25 x).  fp32 graphs meet 1e-5 (test above).  A planned
    budget trains the same function (<= 1e-3 of the all-reside plan)."""
    g = graphs.config_graph(name)
    ol, og = _oracle(g)
    _, ob = _oracle(g, storage="bf16")
    loss, grads, S, P = _run(g)
    assert abs(loss - ol) <= 2e-2 * abs(ol)
    e_gpu, e_ref = rel_errs(grads, og), rel_errs(ob, og)
    print(name, "gpu vs fp64: global", global_rel_err(grads, og), "bf16 reading vs fp64:", global_rel_err(ob, og))
    bad = {k: (e_gpu[k], e_ref[k]) for k in e_gpu if e_gpu[k] > max(2e-2, 1.5 * e_ref[k])}
    assert not bad, bad
    assert global_rel_err(grads, og) <= max(2e-2, 1.25 * global_rel_err(ob, og))
    base = P.stats()
    for frac in (3, 4, 5, 6, 7):
        budget = base["static_bytes"] + (base["peak_extent"] - base["static_bytes"]) * frac // 10
        try:
            tsplit.Plan.plan(tsplit.Graph(g), budget)
            break
        except tsplit.TsError:
            continue
    l2, g2, S2, P2 = _run(g, budget=budget)
    st = P2.stats()
    assert st["peak_extent"] <= budget and st["n_split_tensors"] + st["n_swap_tensors"] > 0
    assert S2.trace() == P2.trace()
    print(name, "budget", frac, "/10: split-vs-unsplit", global_rel_err(g2, grads))
    assert global_rel_err(g2, grads) <= 1e-3
