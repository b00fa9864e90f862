"""End-to-end parity of the CUDA path (C ABI session) against the fp64 oracle and
against itself under different plans (north_star targets:
fp32 <= 1e-5, bf16 <= 2e-2 vs the oracle, split vs unsplit <= 1e-6 for fp32)."""

import random

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from conftest import assert_bf16_parity, global_rel_err, rel_errs  # noqa: E402
from oracle import brute, net, sim  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def _run(g, plan_cfg=None, budget=None, graph_mode=True, on_host=False):
    G = tsplit.Graph(g)
    if budget is not None:
        P = tsplit.Plan.plan(G, budget)
    else:
        P = tsplit.Plan.default(G)
        if plan_cfg and any(len(c) > 3 for c in plan_cfg.values()):  # channel splits: one validated batch
            P.set_many(plan_cfg)
        else:
            for t, (o, p, lead) in (plan_cfg or {}).items():
                P.set(t, o, p, lead)
    S = tsplit.Session(G, P, use_cuda_graph=graph_mode)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    S.set_params(params)
    dev = tsplit.inputs_to_device(G, inputs, pinned_host=on_host)
    loss = S.step(dev)
    return loss, S.grads(), S, P


def _run_unfused(g, **kw):
    """_run with the session's peephole fusions (D-FUSE, D-QKV) off: which fusions apply
    depends on the plan's allocations, and the fused q/k/v backward rounds dX to bf16 once
    instead of three times, so plan invariance is checked with both programs unfused."""
    import os
    os.environ["TSPLIT_NO_FUSION"] = "1"
    try:
        return _run(g, **kw)
    finally:
        os.environ.pop("TSPLIT_NO_FUSION", None)


def _oracle(g):
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    loss, pg, _, _ = net.train_step(g, params, inputs)
    return loss, pg


def test_config1_mlp_fp32_forced_plan_parity():
    """Config 1: 2-way batch split on every op + one swapped activation, fp32."""
    g = graphs.mlp()
    names = {t["name"]: t["id"] for t in g["tensors"]}
    cfg = {t: (tsplit.RESIDE, 2, 1) for t in brute.act_tensors(g)}
    cfg[names["relu0"]] = (tsplit.SWAP, 2, 1)
    loss, grads, S, P = _run(g, cfg)
    st = P.stats()
    assert st["d2h_bytes"] == st["h2d_bytes"] > 0
    ol, og = _oracle(g)
    assert abs(loss - ol) <= 1e-5 * abs(ol)
    errs = rel_errs(grads, og)
    assert max(errs.values()) <= 1e-5, errs
    # split + swap vs unsplit on the GPU
    l0, g0, _, _ = _run(g)
    assert max(rel_errs(grads, g0).values()) <= 1e-6
    # the runtime's allocation trace is the simulator's
    assert S.trace() == [tuple(e) for e in sim.simulate(g, {**sim.default_cfg(g), **cfg}).trace]


@pytest.mark.parametrize("seed", range(3))
def test_bert_tiny_fp32_random_plans(seed):
    g = graphs.config_graph("bert_tiny", dtype="f32")
    r = random.Random(seed)
    cfg = {t: (r.choice([0, 1, 2]), r.choice([1, 2, 4]), r.choice([1, 2])) for t in brute.act_tensors(g)}
    loss, grads, S, P = _run(g, cfg)
    ol, og = _oracle(g)
    assert abs(loss - ol) <= 1e-5 * abs(ol)
    errs = rel_errs(grads, og)
    assert max(errs.values()) <= 1e-5, sorted(errs.items(), key=lambda kv: -kv[1])[:5]
    l0, g0, _, _ = _run(g)
    e0 = rel_errs(grads, g0)
    assert max(e0.values()) <= 1e-6, sorted(e0.items(), key=lambda kv: -kv[1])[:5]


@pytest.mark.parametrize("fused_attention", [False, True])
def test_bert_small_bf16_parity_and_budget(fused_attention):
    """bf16 (R17, D-TOL): every parameter gradient within 2e-2 (per-tensor relative L2) of
    the plain fp64 oracle, unbudgeted and under a planned 40 % budget; with the peephole
    fusions off in both, the budgeted plan computes the all-reside plan's gradients
    (<= 1e-6: splits change only fp32 accumulation order)."""
    g = graphs.config_graph("bert_small", fused_attention=fused_attention)
    ol, og = _oracle(g)
    loss, grads, S, P = _run(g)
    assert abs(loss - ol) <= 2e-2 * abs(ol)
    assert_bf16_parity(grads, og)
    base = P.stats()
    budget = base["static_bytes"] + (base["peak_extent"] - base["static_bytes"]) * 4 // 10
    l2, g2, S2, P2 = _run(g, budget=budget)
    st = P2.stats()
    assert st["peak_extent"] <= budget and st["n_split_tensors"] + st["n_swap_tensors"] + st["n_recompute_tensors"] > 0
    assert S2.trace() == P2.trace()
    assert_bf16_parity(g2, og)
    _, u0, _, _ = _run_unfused(g)
    _, u2, _, _ = _run_unfused(g, budget=budget)
    assert global_rel_err(u2, u0) <= 1e-6


def test_eager_equals_graph_and_host_inputs():
    g = graphs.config_graph("bert_tiny", dtype="f32")
    l1, g1, _, _ = _run(g, graph_mode=True)
    l2, g2, _, _ = _run(g, graph_mode=False, on_host=True)
    assert abs(l1 - l2) <= 1e-6 * abs(l1)
    assert max(rel_errs(g2, g1).values()) <= 1e-6


def test_sgd_step_changes_params_and_loss_drops():
    g = graphs.mlp()
    G = tsplit.Graph(g)
    P = tsplit.Plan.default(G)
    S = tsplit.Session(G, P, lr=0.5)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    S.set_params(params)
    dev = tsplit.inputs_to_device(G, inputs)
    losses = [S.step(dev) for _ in range(5)]
    assert losses[-1] < losses[0]
    assert not np.allclose(S.param("fc0.w"), params["fc0.w"])


def test_bert_large_full_size_properties():
    """BERT-Large b32 s512 at the bench's 25% budget (properties that hold at any size):
    the budgeted plan trains the same function as the all-reside plan (T1 on the GPU),
    the runtime trace is the simulator's, the pool never exceeds the budget, and the
    initial loss is the 2-class chance level ln 2."""
    import math
    g = graphs.config_graph("bert_large")
    G = tsplit.Graph(g)
    base = tsplit.Plan.default(G)
    st = base.stats()
    budget = st["static_bytes"] + (st["peak_extent"] - st["static_bytes"]) // 4
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    dev = tsplit.inputs_to_device(G, inputs)
    P = tsplit.Plan.plan(G, budget)
    assert P.stats()["peak_extent"] <= budget
    S = tsplit.Session(G, P, slab_bytes=budget)
    S.set_params(params)
    l_b = S.step(dev)
    g_b = S.grads()
    assert S.trace() == P.trace()
    del S
    torch.cuda.empty_cache()
    S0 = tsplit.Session(G, base)
    S0.set_params(params)
    l_0 = S0.step(dev)
    g_0 = S0.grads()
    del S0
    torch.cuda.empty_cache()
    assert abs(l_b - math.log(2.0)) < 0.05 and abs(l_0 - l_b) <= 1e-3 * abs(l_0)
    assert all(np.isfinite(v).all() for v in g_b.values())
    assert global_rel_err(g_b, g_0) <= 1e-3


def test_nccl_bucketed_allreduce_single_rank():
    """The data-parallel path (per-bucket ncclAllReduce on the comm stream, captured in
    the CUDA graph, SGD after the last bucket) with a 1-rank communicator: gradients
    and the updated parameters equal the communicator-free session's."""
    g = graphs.config_graph("bert_tiny", dtype="f32")
    G = tsplit.Graph(g)
    P = tsplit.Plan.default(G)
    comm = tsplit.nccl_comm(0, 1, lambda b: b)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    dev = tsplit.inputs_to_device(G, inputs)
    out = []
    for c in (None, comm):
        S = tsplit.Session(G, P, lr=0.1, nccl_comm=c, world_size=1)
        S.set_params(params)
        S.step(dev)
        S.step(dev)
        out.append((S.grads(), S.param("l0.ffn1.w")))
    assert len(P.grad_buckets()) >= 1
    # equal up to the run-to-run order of fp32 atomics (embedding rows, split-K partials),
    # which after one SGD step also perturbs the second step's tiny-norm tensors
    assert global_rel_err(out[1][0], out[0][0]) <= 1e-6
    assert max(rel_errs(out[1][0], out[0][0]).values()) <= 1e-4
    assert np.allclose(out[1][1], out[0][1], rtol=1e-6, atol=1e-9)


def test_nccl_bf16_gradient_buckets_single_rank():
    """bf16 gradient buckets (ts_session_cfg.grad_allreduce_bf16): each bucket is
    rounded to bf16, summed by ncclAllReduce in bf16 and widened back.  With a 1-rank
    communicator the sum is the identity, so every gradient equals the fp32-bucket session's
    rounded to bf16, bit for bit (lr = 0: both sessions read the same parameters)."""
    import torch
    g = graphs.config_graph("bert_tiny", dtype="f32")
    G = tsplit.Graph(g)
    P = tsplit.Plan.default(G)
    comm = tsplit.nccl_comm(0, 1, lambda b: b)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    dev = tsplit.inputs_to_device(G, inputs)
    out = []
    for bf in (False, True):
        S = tsplit.Session(G, P, lr=0.0, nccl_comm=comm, world_size=1, grad_allreduce_bf16=bf)
        S.set_params(params)
        S.step(dev)
        out.append(S.grads())
    for k, v in out[0].items():
        want = torch.from_numpy(np.asarray(v, np.float32)).to(torch.bfloat16).float().numpy()
        assert np.array_equal(out[1][k], want), k


def _fusion_pair(g, cfg, var="TSPLIT_NO_FUSION", qkv=False):
    """The same step with and without a session fusion: `var` = 1 turns it off.  The
    linear + gelu comparison keeps the q/k/v grouping off in both runs (qkv=False)."""
    import os
    out = []
    for off in ("1", "0"):
        os.environ[var] = off
        if not qkv:
            os.environ["TSPLIT_NO_QKV_FUSION"] = "1"
        try:
            loss, grads, S, _ = _run(g, cfg)
            out.append((loss, grads, S.launches()))
        finally:
            os.environ.pop(var, None)
            os.environ.pop("TSPLIT_NO_QKV_FUSION", None)
    return out


@pytest.mark.parametrize("plan", ["reside", "recompute_qkv", "split"])
def test_qkv_grouped_fusion(plan):
    """bf16 graphs (reading D-QKV): the q/k/v linear micro-ops of a layer run as grouped
    GEMMs — forward and recompute replays one N-grouped product, backward one K-grouped dX
    (summed in fp32, a single accumulation into dX) and one M-grouped dW.  The forward is
    the same arithmetic (loss bit-identical); the backward differs only by the bf16
    rounding of the dX accumulation; both stay within the bf16 bar of the oracle."""
    g = graphs.config_graph("bert_small", fused_attention=True)
    names = {t["name"]: t["id"] for t in g["tensors"]}
    cfg = {}
    if plan == "recompute_qkv":
        cfg = {names[f"l0.{x}"]: (tsplit.RECOMPUTE, 1, 1) for x in ("q", "k", "v")}
    elif plan == "split":
        cfg = {names[f"l1.{x}"]: (tsplit.RESIDE, 2, 1) for x in ("q", "k", "v")}
    (l0, g0, n0), (l1, g1, n1) = _fusion_pair(g, cfg, var="TSPLIT_NO_QKV_FUSION", qkv=True)
    assert n1 < n0, (n0, n1)
    assert l1 == l0
    assert global_rel_err(g1, g0) <= 5e-3
    assert_bf16_parity(g1, _oracle(g)[1])


@pytest.mark.parametrize("fused_attention", [False, True])
@pytest.mark.parametrize("plan", ["reside", "recompute_ffn", "split_swap"])
def test_linear_gelu_fusion_equals_unfused(fused_attention, plan):
    """bf16 graphs: the FFN1 GEMM epilogue writes U and gelu(U), and the FFN2 dX GEMM
    writes dU = dH * gelu'(U) directly, where the plan leaves the ranges free
    (session.cu build_program).  The fused program computes what the unfused one does —
    the epilogue rounds through bf16 exactly where the separate kernels store — and
    launches fewer kernels; it also stays within the bf16 bar of the fp64 oracle."""
    g = graphs.config_graph("bert_small", fused_attention=fused_attention)
    names = {t["name"]: t["id"] for t in g["tensors"]}
    cfg = {}
    if plan == "recompute_ffn":  # replays R(ffn1), R(gelu) are adjacent too
        cfg = {names["l0.ffn1"]: (tsplit.RECOMPUTE, 1, 1), names["l0.gelu"]: (tsplit.RECOMPUTE, 1, 1),
               names["l1.gelu"]: (tsplit.RECOMPUTE, 1, 1)}
    elif plan == "split_swap":  # split pieces are not fused (P > 1), swapped ones still are
        cfg = {names["l0.ffn1"]: (tsplit.RESIDE, 2, 1), names["l0.gelu"]: (tsplit.RESIDE, 2, 1),
               names["l1.ffn1"]: (tsplit.SWAP, 1, 1)}
    (l0, g0, n0), (l1, g1, n1) = _fusion_pair(g, cfg)
    assert n1 < n0, (n0, n1)
    assert abs(l1 - l0) <= 1e-6 * abs(l0)
    assert global_rel_err(g1, g0) <= 1e-6
    assert_bf16_parity(g1, _oracle(g)[1])


@pytest.mark.parametrize("cache", [1 << 20, 2 ** 64 - 1])
def test_lru_recompute_cache_session(cache):
    """D-LRU recompute cache on the GPU: fewer replays, the runtime's allocation trace is
    the simulator's (regenerated pieces held across backward groups), and the gradients
    equal the memory-centric plan's (fp32: 1e-6) and the oracle's (1e-5)."""
    g = graphs.config_graph("bert_tiny", dtype="f32", fused_attention=True)
    names = {t["name"]: t["id"] for t in g["tensors"]}
    cfg = {names[f"l{i}.{x}"]: (tsplit.RECOMPUTE, 1, 1) for i in (0, 1) for x in ("ffn1", "gelu", "ln1", "q", "k")}
    cfg[names["l0.v"]] = (tsplit.RECOMPUTE, 2, 1)
    G = tsplit.Graph(g)
    out = []
    for c in (0, cache):
        P = tsplit.Plan.default(G)
        for t, (o, p, lead) in cfg.items():
            P.set(t, o, p, lead)
        P.set_recompute_cache(c)
        S = tsplit.Session(G, P)
        params, inputs = gen.init_params(g), gen.make_inputs(g)
        S.set_params(params)
        loss = S.step(tsplit.inputs_to_device(G, inputs))
        assert S.trace() == [tuple(e) for e in sim.simulate(g, {**sim.default_cfg(g), **cfg}, cache_bytes=c).trace]
        out.append((loss, S.grads(), P.stats()["n_replay"]))
    assert out[1][2] < out[0][2]
    assert max(rel_errs(out[1][1], out[0][1]).values()) <= 1e-6
    ol, og = _oracle(g)
    assert max(rel_errs(out[1][1], og).values()) <= 1e-5


def test_bert_large_shaped_layer_bf16_parity():
    """A BERT-Large-shaped encoder layer (hidden 1024, 16 heads, seq 512, batch 4, the real
    vocabulary; fused attention, dropout 0.1) under a plan with sample splits, a swap and
    recomputes, against the plain fp64 oracle per tensor (north_star bf16 bar, R17)."""
    g = graphs.config_graph("bert_large", layers=1, batch=4, fused_attention=True)
    names = {t["name"]: t["id"] for t in g["tensors"]}
    cfg = {names["l0.ln1"]: (tsplit.RECOMPUTE, 2, 1), names["l0.ffn1"]: (tsplit.RESIDE, 2, 1),
           names["l0.gelu"]: (tsplit.SWAP, 2, 1), names["l0.q"]: (tsplit.RECOMPUTE, 1, 1),
           names["l0.k"]: (tsplit.RECOMPUTE, 1, 1), names["l0.ctx"]: (tsplit.SWAP, 1, 2),
           names["l0.res2"]: (tsplit.RESIDE, 4, 1)}
    loss, grads, S, P = _run(g, cfg)
    st = P.stats()
    assert st["n_split_tensors"] > 0 and st["n_swap_tensors"] > 0 and st["n_recompute_tensors"] > 0
    assert S.trace() == [tuple(e) for e in sim.simulate(g, {**sim.default_cfg(g), **cfg}).trace]
    ol, og = _oracle(g)
    assert abs(loss - ol) <= 2e-2 * abs(ol)
    errs = assert_bf16_parity(grads, og)
    print("bert-large-shaped layer: worst", sorted(errs.items(), key=lambda kv: -kv[1])[:4])
    _, g0, _, _ = _run(g)
    assert global_rel_err(grads, g0) <= 1e-3


@pytest.mark.parametrize("fused_attention", [False, True])
@pytest.mark.parametrize("graph_mode", [True, False])
def test_dropout_masks_follow_the_step_counter(fused_attention, graph_mode):
    """R15 / D-RNG: the dropout masks of step k use Philox counter word `step` = k.  The
    session keeps the step in device memory and advances it at the end of every step, so a
    captured CUDA graph replays with the live value.  Three steps with lr = 0 (parameters
    fixed) give gradients equal to the oracle's `train_step(step=k)` for k = 0, 1, 2 — and
    different from one another (the masks change)."""
    g = graphs.config_graph("bert_tiny", dtype="f32", fused_attention=fused_attention)
    G = tsplit.Graph(g)
    P = tsplit.Plan.default(G)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    S = tsplit.Session(G, P, use_cuda_graph=graph_mode, lr=0.0)
    S.set_params(params)
    dev = tsplit.inputs_to_device(G, inputs)
    prev = None
    for k in range(3):
        loss = S.step(dev)
        grads = S.grads()
        ol, og, _, _ = net.train_step(g, params, inputs, step=k)
        assert abs(loss - ol) <= 1e-5 * abs(ol), (k, loss, ol)
        errs = rel_errs(grads, og)
        assert max(errs.values()) <= 1e-5, (k, sorted(errs.items(), key=lambda kv: -kv[1])[:3])
        if prev is not None:
            assert global_rel_err(grads, prev) > 1e-3  # a new mask, not a replayed one
        prev = grads


@pytest.mark.parametrize("seed", range(3))
def test_bert_small_bf16_random_plans(seed):
    """bf16 graphs under random split / swap / recompute plans (the fused-attention graph:
    its f32 / i32 auxiliary outputs are then read through sub-views of other sizes): per
    tensor within 2e-2 of the plain fp64 oracle, and — with the peephole fusions off in
    both — equal to the all-reside plan up to fp32 accumulation order.  In a bf16 graph a
    reordered fp32 sum (a different GEMM split-K, dW summed over micro-ops) moves a stored
    value across a bf16 rounding boundary now and then — a one-ulp (2^-8) change that the
    rest of the backward carries along: measured 6e-5 .. 3e-4 over these plans, bar 1e-3
    globally, the full-size BERT-Large one (the fp32 graphs' 1e-6 is that of fp32
    storage, where the same plans are checked bit-for-bit-level)."""
    g = graphs.config_graph("bert_small", fused_attention=True)
    r = random.Random(300 + seed)
    cfg = {t: (r.choice([0, 1, 2]), r.choice([1, 2, 4]), r.choice([1, 2])) for t in brute.act_tensors(g)}
    loss, grads, S, P = _run(g, cfg)
    assert S.trace() == [tuple(e) for e in sim.simulate(g, {**sim.default_cfg(g), **cfg}).trace]
    ol, og = _oracle(g)
    assert abs(loss - ol) <= 2e-2 * abs(ol)
    assert_bf16_parity(grads, og)
    _, u1, _, _ = _run_unfused(g, plan_cfg=cfg)
    _, u0, _, _ = _run_unfused(g)
    assert global_rel_err(u1, u0) <= 1e-3


def test_profile_measure_times_every_split_width():
    """a2 ("profiles every single operation before training", P:L281 cudaEvent,
    P:L125 Fig. 5): ts_profile_measure times every op's forward and backward at p = 1, 2,
    4, 8 (batch 8 bounds the sample split), with the per-micro-op degradation the planner
    must see — the GEMM-heavy ops cost more as 8 micro-ops than as one — and measures the
    pinned PCIe bandwidth; the planner plans with it."""
    g = graphs.config_graph("bert_small", fused_attention=True)
    G = tsplit.Graph(g)
    dev = tsplit.inputs_to_device(G, gen.make_inputs(g))
    prof = tsplit.Profile.measure(G, dev, max_p=16)
    ana = tsplit.Profile(G)
    names = [o["name"] for o in g["ops"]]
    for o, op in enumerate(g["ops"]):
        for p in (1, 2, 4, 8):
            f, b = prof.get(o, p)
            assert f > 0, (op["name"], p)
            assert prof.get(o, p) != ana.get(o, p)  # measured, not the analytic model
    ffn = [names.index(f"l{i}.ffn{j}") for i in range(2) for j in (1, 2)]
    slower = [sum(prof.get(o, 8)) > sum(prof.get(o, 1)) for o in ffn]
    assert all(slower), [(names[o], prof.get(o, 1), prof.get(o, 8)) for o in ffn]
    d2h, h2d = prof.pcie()
    assert 5e9 < d2h < 2e11 and 5e9 < h2d < 2e11, (d2h, h2d)
    base = tsplit.Plan.default(G).stats()
    budget = base["static_bytes"] + (base["peak_extent"] - base["static_bytes"]) // 3
    P = tsplit.Plan.plan(G, budget, profile=prof)
    assert P.stats()["peak_extent"] <= budget
