"""f4 (§VI-D): a planned augmented graph exported to
a standalone stock-PyTorch module computes the unsplit step — T1 through another
framework.  CPU: the exported module in float64 against the fp64 oracle under random
split / swap / recompute plans (and LRU recompute caches) of every graph family; GPU: the
exported module on cuda against the C-ABI session under the same plan."""

import importlib.util
import os
import random

import numpy as np
import pytest

torch = pytest.importorskip("torch")

from conftest import assert_bf16_parity, rel_errs  # noqa: E402
from oracle import brute, net  # noqa: E402
from paper_conf_icde_niemyc22_b200 import export, tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def _load(path):
    spec = importlib.util.spec_from_file_location(os.path.basename(path)[:-3], path)
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    return mod


def _random_plan(g, G, seed, cache=0):
    P = tsplit.Plan.default(G)
    r = random.Random(seed)
    for t in brute.act_tensors(g):
        P.set(t, r.choice([0, 1, 2]), r.choice([1, 2, 4]), r.choice([1, 2]))
    if cache:
        P.set_recompute_cache(cache)
    return P


CASES = [("mlp", {}), ("bert_tiny", dict(dtype="f32")), ("bert_tiny", dict(dtype="f32", fused_attention=True)),
         ("vgg_tiny", dict(dtype="f32")), ("resnet_tiny", dict(dtype="f32")),
         ("transformer_tiny", dict(dtype="f32", seq=32))]


@pytest.mark.parametrize("case", range(len(CASES)))
@pytest.mark.parametrize("seed", range(2))
def test_exported_step_equals_the_oracle(case, seed, tmp_path):
    name, kw = CASES[case]
    g = graphs.config_graph(name, **kw)
    G = tsplit.Graph(g)
    P = _random_plan(g, G, 10 * case + seed, cache=(0 if seed == 0 else 4096))
    st = P.stats()
    mod = _load(export.export_torch(G, P, str(tmp_path / f"step_{case}_{seed}.py")))
    src = open(mod.__file__).read()
    assert "paper_conf_icde_niemyc22_b200" not in src.split('"""', 2)[2]  # standalone: torch only
    assert "import torch" in src
    assert len(mod.ITEMS) == st["n_items"]
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    loss, grads = mod.AugmentedStep("cpu", torch.float64)(params, inputs)
    ol, og, _, _ = net.train_step(g, params, inputs)
    assert abs(loss - ol) <= 1e-12 * abs(ol)
    errs = rel_errs({k: v.numpy() for k, v in grads.items()}, og)
    assert max(errs.values()) <= 1e-12, sorted(errs.items(), key=lambda kv: -kv[1])[:3]


SPLIT_CASES = [("mlp", "chan2"), ("bert_tiny", "chan2"), ("vgg_tiny", "band"), ("resnet_tiny", "band"),
               ("vgg_tiny", "chan4"), ("resnet_tiny", "chan4")]


@pytest.mark.parametrize("case", range(len(SPLIT_CASES)))
def test_exported_channel_and_band_plans_equal_the_oracle(case, tmp_path):
    """Channel (D-CH: 2-D and image blocks) and height / width band (D-ATTR: staged halo
    rectangles) plans exported to torch: the fp64 module equals the fp64 oracle."""
    from test_oracle_attr import _rand_attr_cfg
    from test_oracle_channel import CHAINS, channel_cfg
    from test_oracle_channel4 import rand_chan4_cfg
    name, kind = SPLIT_CASES[case]
    g = graphs.config_graph(name, **({} if name == "mlp" else {"dtype": "f32"}))
    r = random.Random(40 + case)
    cfg = (channel_cfg(g, r, CHAINS[name], prob=0.9) if kind == "chan2" else
           _rand_attr_cfg(g, r) if kind == "band" else rand_chan4_cfg(g, r))
    G = tsplit.Graph(g)
    P = tsplit.Plan.default(G)
    P.set_many({t: cfg[t] for t in brute.act_tensors(g)})
    mod = _load(export.export_torch(G, P, str(tmp_path / f"split_{case}.py")))
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    loss, grads = mod.AugmentedStep("cpu", torch.float64)(params, inputs)
    ol, og, _, _ = net.train_step(g, params, inputs)
    assert abs(loss - ol) <= 1e-12 * abs(ol)
    errs = rel_errs({k: v.numpy() for k, v in grads.items()}, og)
    assert max(errs.values()) <= 1e-12, sorted(errs.items(), key=lambda kv: -kv[1])[:3]


@pytest.mark.gpu
@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_exported_step_on_cuda_matches_the_session(dtype, tmp_path):
    """The exported module on the GPU (torch kernels, swaps through pinned host tensors on
    side streams) and the C-ABI session (own kernels) run the same planned bert step: fp32
    within 1e-5 of each other and of the oracle; bf16 both within the bf16 bar."""
    g = graphs.config_graph("bert_tiny" if dtype == "f32" else "bert_small", dtype=dtype, fused_attention=True)
    G = tsplit.Graph(g)
    base = tsplit.Plan.default(G).stats()
    budget = base["static_bytes"] + (base["peak_extent"] - base["static_bytes"]) * 4 // 10
    P = tsplit.Plan.plan(G, budget)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    mod = _load(export.export_torch(G, P, str(tmp_path / f"step_gpu_{dtype}.py")))
    torch.backends.cuda.matmul.allow_tf32 = False
    torch.backends.cudnn.allow_tf32 = False
    loss, grads = mod.AugmentedStep("cuda", torch.float32 if dtype == "f32" else torch.bfloat16)(params, inputs)
    grads = {k: v.float().cpu().numpy() for k, v in grads.items()}
    S = tsplit.Session(G, P)
    S.set_params(params)
    ls = S.step(tsplit.inputs_to_device(G, inputs))
    gs = S.grads()
    ol, og, _, _ = net.train_step(g, params, inputs)
    if dtype == "f32":
        assert max(rel_errs(grads, og).values()) <= 1e-5
        assert max(rel_errs(grads, gs).values()) <= 1e-5
        assert abs(loss - ls) <= 1e-5 * abs(ls)
    else:
        assert_bf16_parity(grads, og)
        assert_bf16_parity(gs, og)
