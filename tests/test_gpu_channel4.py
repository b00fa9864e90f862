"""Channel splits of NHWC images on the GPU (reading D-CH, 4-D part): conv2d in
channel mode (weight rows / bias block k), channel-local ReLU / add / batch norm (per-block
statistics) / max pooling, a conv reading every block through a staged merge; whole steps of
the tiny / small VGG and ResNet graphs under random plans against the fp64 oracle and the
unsplit GPU step, and the session's trace against the simulator's."""

import random

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from conftest import global_rel_err, rel_errs  # noqa: E402
from oracle import brute, net, sim  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from test_oracle_channel4 import rand_chan4_cfg  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def _run(g, cfg=None):
    G = tsplit.Graph(g)
    P = tsplit.Plan.default(G)
    if cfg:
        P.set_many({t: cfg[t] for t in brute.act_tensors(g)})
    S = tsplit.Session(G, P)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    S.set_params(params)
    loss = S.step(tsplit.inputs_to_device(G, inputs))
    return loss, S.grads(), S, P


@pytest.mark.parametrize("name", ["vgg_tiny", "resnet_tiny"])
@pytest.mark.parametrize("seed", range(3))
def test_channel4_plans_fp32(name, seed):
    g = graphs.config_graph(name, dtype="f32")
    cfg = rand_chan4_cfg(g, random.Random(600 + seed), min_block=4)
    loss, grads, S, P = _run(g, cfg)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    ol, og, _, _ = net.train_step(g, params, inputs)
    assert abs(loss - ol) <= 1e-5 * abs(ol)
    errs = rel_errs(grads, og)
    assert max(errs.values()) <= 1e-5, sorted(errs.items(), key=lambda kv: -kv[1])[:5]
    l0, g0, _, _ = _run(g)
    e0 = rel_errs(grads, g0)
    assert max(e0.values()) <= 3e-6, sorted(e0.items(), key=lambda kv: -kv[1])[:5]
    assert S.trace() == [tuple(e) for e in sim.simulate(g, cfg).trace]


@pytest.mark.parametrize("name", ["vgg_small", "resnet_small"])
@pytest.mark.parametrize("seed", range(2))
def test_channel4_plans_bf16(name, seed):
    """bf16: the D-TOL-CNN bar against the fp64 oracle, and within 1e-2 of the unsplit step."""
    g = graphs.config_graph(name)
    cfg = rand_chan4_cfg(g, random.Random(700 + seed), min_block=8)
    loss, grads, S, P = _run(g, cfg)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    ol, og, _, _ = net.train_step(g, params, inputs)
    _, ob, _, _ = net.train_step(g, params, inputs, storage="bf16")
    e_gpu, e_ref = rel_errs(grads, og), rel_errs(ob, og)
    bad = {k: (e_gpu[k], e_ref[k]) for k in e_gpu if e_gpu[k] > max(2e-2, 1.5 * e_ref[k])}
    assert not bad, bad
    assert global_rel_err(grads, og) <= max(2e-2, 1.25 * global_rel_err(ob, og))
    l0, g0, _, _ = _run(g)
    print(name, seed, "channel vs unsplit", global_rel_err(grads, g0))
    assert abs(loss - l0) <= 1e-3 * abs(l0)
    assert global_rel_err(grads, g0) <= 1e-2
    assert S.trace() == [tuple(e) for e in sim.simulate(g, cfg).trace]
