"""Channel (parameter-dim) splits on the GPU (reading D-CH, Fig. 6): linear
micro-ops over output-channel blocks (weight rows / bias blocks), elementwise micro-ops
over column blocks, and linears reading a column-blocked X (K blocks summed), with swap
and recompute of individual blocks.  Parity against the fp64 oracle, against unsplit GPU
execution, and the runtime trace against the simulator."""
import random

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from conftest import assert_bf16_parity, rel_errs  # noqa: E402
from oracle import brute, net, sim  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from test_gpu_session import _oracle, _run  # noqa: E402
from test_oracle_channel import CHAINS, channel_cfg  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def _full(g, cfg):
    return {**sim.default_cfg(g), **cfg}


def test_mlp_fp32_channel_split_swap_recompute():
    """Config 1 shape with fc0 -> relu0 in 4 column blocks (relu0 swapped block by block)
    and fc1 -> relu1 in 2 blocks recomputed: fp32 parity <= 1e-5 vs the oracle, <= 1e-6
    vs unsplit GPU execution, trace = simulator."""
    g = graphs.mlp()
    names = {t["name"]: t["id"] for t in g["tensors"]}
    cfg = {t: (tsplit.RESIDE, 1, 1) for t in brute.act_tensors(g)}
    cfg[names["fc0"]] = (tsplit.RESIDE, 4, 1, 1)
    cfg[names["relu0"]] = (tsplit.SWAP, 4, 1, 1)
    cfg[names["fc1"]] = (tsplit.RECOMPUTE, 2, 1, 1)
    cfg[names["relu1"]] = (tsplit.RECOMPUTE, 2, 1, 1)
    loss, grads, S, P = _run(g, cfg)
    st = P.stats()
    assert st["d2h_bytes"] == st["h2d_bytes"] > 0 and st["n_replay"] > 0
    ol, og = _oracle(g)
    assert abs(loss - ol) <= 1e-5 * abs(ol)
    assert max(rel_errs(grads, og).values()) <= 1e-5
    l0, g0, _, _ = _run(g)
    assert max(rel_errs(grads, g0).values()) <= 1e-6
    assert S.trace() == [tuple(e) for e in sim.simulate(g, _full(g, cfg)).trace]


@pytest.mark.parametrize("seed", range(4))
def test_mlp_fp32_random_channel_plans(seed):
    g = graphs.mlp()
    cfg = channel_cfg(g, random.Random(200 + seed), CHAINS["mlp"], prob=0.9)
    loss, grads, S, P = _run(g, cfg)
    ol, og = _oracle(g)
    assert abs(loss - ol) <= 1e-5 * abs(ol)
    assert max(rel_errs(grads, og).values()) <= 1e-5
    assert S.trace() == [tuple(e) for e in sim.simulate(g, cfg).trace]


@pytest.mark.parametrize("dtype", ["f32", "bf16"])
def test_bert_ffn_channel_split(dtype):
    """BERT FFN (ffn1 -> gelu) in column blocks; ffn2 reads the blocks as K slices
    (bert_tiny in fp32, bert_small — the bf16 parity size — in bf16)."""
    g = graphs.config_graph("bert_tiny" if dtype == "f32" else "bert_small", dtype=dtype)
    names = {t["name"]: t["id"] for t in g["tensors"]}
    cfg = {names["l0.ffn1"]: (tsplit.RECOMPUTE, 4, 1, 1), names["l0.gelu"]: (tsplit.SWAP, 4, 1, 1),
           names["l1.ffn1"]: (tsplit.RESIDE, 2, 1, 1), names["l1.gelu"]: (tsplit.RECOMPUTE, 2, 1, 1)}
    loss, grads, S, P = _run(g, cfg)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    if dtype == "f32":
        ol, og = _oracle(g)
        assert abs(loss - ol) <= 1e-5 * abs(ol)
        assert max(rel_errs(grads, og).values()) <= 1e-5
        l0, g0, _, _ = _run(g)
        assert max(rel_errs(grads, g0).values()) <= 1e-6
    else:
        _, og, _, _ = net.train_step(g, params, inputs)
        assert_bf16_parity(grads, og)
    assert S.trace() == [tuple(e) for e in sim.simulate(g, _full(g, cfg)).trace]


def test_planned_channel_split_batch1_mlp():
    """Alg. 2 at batch 1 chooses parameter-dim splits (D-CH); the GPU step under that plan
    matches the fp64 oracle (fp32 <= 1e-5) and the runtime trace is the planned one."""
    g = graphs.mlp(batch=1, in_dim=64, hidden=2048, depth=3, classes=10)
    G = tsplit.Graph(g)
    st = tsplit.Plan.default(G).stats()
    budget = st["static_bytes"] + int(0.75 * (st["peak_extent"] - st["static_bytes"]))
    loss, grads, S, P = _run(g, budget=budget)
    assert any(P.get_dim(t) == 1 for t in brute.act_tensors(g))
    ol, og = _oracle(g)
    assert abs(loss - ol) <= 1e-5 * abs(ol)
    assert max(rel_errs(grads, og).values()) <= 1e-5
    assert S.trace() == P.trace()
