"""The bf16 precision's own distance from fp64 (readings D-TOL / D-TOL-CNN),
measured with the oracle alone — no GPU, no product code.

`net.train_step(storage="bf16")` rounds every stored activation and activation gradient
to bf16 (pinned against torch's conversion in test_oracle_ops.py) and keeps fp64
arithmetic otherwise, so its distance from the plain fp64 step is a lower-order estimate
of what *any* bf16-storage implementation carries.  These facts decide which bf16 bar a
GPU test can honestly hold:

* BERT at the parity size (bert_small: hidden 256, seq 128, batch 8): every tensor is
  within 1.5e-2, so the north_star bar (2e-2 per tensor) is attainable and the GPU tests
  hold it against the plain oracle.
* ReLU CNNs (vgg_small / resnet_small): the early conv / BN gradients are 5-25 % away,
  because rounding the forward values flips ReLU and max-pool decisions (a perturbation of
  fp32 size, 2^-24, moves the same gradients by < 1e-5 — the map is well conditioned; the
  bf16 distance comes from the discrete flips).  No bf16-storage execution meets 2e-2 per
  tensor there; the GPU CNN tests bound the kernels by this distance instead.
"""

import numpy as np
import pytest

from conftest import global_rel_err, rel_errs
from oracle import net
from tsinputs import gen, graphs


def _gap(name, perturb=None):
    g = graphs.config_graph(name)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    _, ref, _, _ = net.train_step(g, params, inputs)
    _, got, _, _ = net.train_step(g, params, inputs, storage="bf16")
    return rel_errs(got, ref), global_rel_err(got, ref)


def test_bert_small_bf16_storage_is_within_the_bar():
    errs, glob = _gap("bert_small")
    assert max(errs.values()) <= 1.5e-2, sorted(errs.items(), key=lambda kv: -kv[1])[:3]
    assert glob <= 1e-2


@pytest.mark.parametrize("name,floor", [("vgg_small", 5e-2), ("resnet_small", 1e-1)])
def test_relu_cnn_bf16_storage_misses_the_bar(name, floor):
    errs, glob = _gap(name)
    assert max(errs.values()) >= floor, sorted(errs.items(), key=lambda kv: -kv[1])[:3]


def test_relu_cnn_gradient_is_well_conditioned_at_fp32_size():
    """Relative forward perturbations of 2^-24 (fp32 rounding size) on every stored value
    move vgg_small's gradients by < 1e-5: the bf16 distance above is the flips, and the
    fp32 bar (1e-5) the fp32 CNN tests hold is the right one for fp32 storage."""
    g = graphs.config_graph("vgg_small")
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    _, ref, _, _ = net.train_step(g, params, inputs)
    r = np.random.default_rng(7)
    val = net.initial_values(g, params, inputs)
    loss_id = next(op["outputs"][0] for op in g["ops"] if op["kind"] == "xent")
    for op in g["ops"]:
        y = net.forward_op(g, op, val)
        val[op["outputs"][0]] = y * (1 + 2.0 ** -24 * r.uniform(-1, 1, np.shape(y))) if op["kind"] != "xent" else y
    ng = net.needs_grad(g)
    grad = {}
    for op in reversed(g["ops"]):
        o = op["outputs"][0]
        if o != loss_id and o not in grad:
            continue
        for tid, gg in net.backward_op(g, op, val, grad.get(o)).items():
            if tid in ng:
                grad[tid] = grad[tid] + gg if tid in grad else gg
    got = {t["name"]: grad[t["id"]] for t in g["tensors"] if t["kind"] == "param"}
    assert max(rel_errs(got, ref).values()) <= 1e-5
