"""Host C++ core (libtsplit.so, no GPU calls) against the oracle simulator:
Alg. 1 order, static region, allocation trace bit for bit, peaks, and the
planner's feasibility (T8)."""

import random

import pytest

from oracle import brute, sim
from paper_conf_icde_niemyc22_b200 import tsplit
from tsinputs import graphs


def _apply(plan, cfg, acts):
    for t in acts:
        c = cfg[t]
        plan.set(t, c[0], c[1], c[2], c[3] if len(c) > 3 else 0, c[4] if len(c) > 4 else 0)


def _compare(g, cfg, cache=0):
    G = tsplit.Graph(g)
    plan = tsplit.Plan.default(G)
    _apply(plan, cfg, brute.act_tensors(g))
    if cache:
        plan.set_recompute_cache(cache)
    ref = sim.simulate(g, cfg, cache_bytes=cache)
    got = plan.trace()
    assert len(got) == len(ref.trace)
    for a, b in zip(got, ref.trace):
        assert a == tuple(b), (a, b)
    st = plan.stats()
    assert st["peak_live"] == ref.peak_live
    assert st["peak_extent"] == ref.peak_extent
    assert st["n_replay"] == ref.n_replay
    assert st["d2h_bytes"] == ref.d2h_bytes and st["h2d_bytes"] == ref.h2d_bytes
    kinds = [it[0] for it in plan.items()]
    assert kinds == [it.kind for it in ref.items]


def test_library_exports_every_declared_symbol():
    L = tsplit.lib()
    names = tsplit.exported_symbols()
    assert len(names) > 30
    missing = [n for n in names if not hasattr(L, n)]
    assert not missing, missing


@pytest.mark.parametrize("gname", ["mlp", "bert_tiny", "bert_large"])
def test_schedule_and_static_match_oracle(gname):
    g = graphs.config_graph(gname)
    G = tsplit.Graph(g)
    assert G.schedule() == sim.schedule(g)
    assert G.static_bytes() == sim.static_bytes(g)


def test_trace_bit_exact_all_plans_tiny_mlp():
    g = graphs.mlp(batch=4, hidden=8, depth=2, in_dim=8, classes=3)
    for cfg in brute.enumerate_plans(g, ps=(1, 2, 4)):
        _compare(g, cfg)


@pytest.mark.parametrize("seed", range(6))
def test_trace_bit_exact_random_plans_bert_tiny(seed):
    g = graphs.config_graph("bert_tiny")
    r = random.Random(seed)
    cfg = sim.default_cfg(g)
    for t in brute.act_tensors(g):
        cfg[t] = (r.choice([0, 1, 2]), r.choice([1, 2, 4]), r.choice([1, 2, 3]))
    _compare(g, cfg)


@pytest.mark.parametrize("gname", ["bert_tiny", "resnet_tiny"])
@pytest.mark.parametrize("seed", range(4))
def test_trace_bit_exact_random_plans_with_release_lags(gname, seed):
    """D-LAG: swapped tensors with release lags 0..12 (the range a swap-out frees returns
    to the pool after that many compute items, before the swap-in) — the C++ expansion
    and pool trace equal the oracle's bit for bit."""
    g = graphs.config_graph(gname)
    r = random.Random(500 + seed)
    cfg = sim.default_cfg(g)
    for t in brute.act_tensors(g):
        o = r.choice([0, 1, 1, 2])
        cfg[t] = (o, r.choice([1, 2, 4]), r.choice([1, 2, 5]), 0, r.choice([0, 1, 3, 12]) if o == 1 else 0)
    _compare(g, cfg)


@pytest.mark.parametrize("seed", range(3))
def test_trace_bit_exact_random_plans_transformer(seed):
    """The encoder-decoder workload (f4): Alg. 1 order, static region and the trace of random
    split / swap / recompute plans (with release lags) equal the oracle simulator's."""
    g = graphs.config_graph("transformer_tiny")
    G = tsplit.Graph(g)
    assert G.schedule() == sim.schedule(g) and G.static_bytes() == sim.static_bytes(g)
    r = random.Random(700 + seed)
    cfg = sim.default_cfg(g)
    for t in brute.act_tensors(g):
        o = r.choice([0, 1, 2])
        cfg[t] = (o, r.choice([1, 2, 4]), r.choice([1, 2]), 0, r.choice([0, 4]) if o == 1 else 0)
    _compare(g, cfg)


def test_default_trace_bert_large():
    g = graphs.config_graph("bert_large")
    _compare(g, sim.default_cfg(g))


def test_config1_forced_plan():
    """Config 1: 2-way batch split on every op plus one swapped activation."""
    g = graphs.mlp()
    cfg = sim.default_cfg(g)
    names = {t["name"]: t["id"] for t in g["tensors"]}
    for t in brute.act_tensors(g):
        cfg[t] = (sim.RESIDE, 2, 1)
    cfg[names["relu0"]] = (sim.SWAP, 2, 1)
    _compare(g, cfg)
    ref = sim.simulate(g, cfg)
    assert ref.d2h_bytes == ref.h2d_bytes == 8 * 256 * 4


def test_plan_serialize_roundtrip():
    g = graphs.config_graph("bert_tiny")
    G = tsplit.Graph(g)
    P = tsplit.Plan.default(G)
    t = G.names["l0.probs"]
    P.set(t, tsplit.RECOMPUTE, 2, 1)
    blob = P.serialize()
    Q = tsplit.Plan.deserialize(G, blob)
    assert Q.trace() == P.trace()
    assert Q.get(t) == (tsplit.RECOMPUTE, 2, 1)


def test_planner_feasible_plans_fit_and_simulate_exactly():
    g = graphs.config_graph("bert_tiny")
    G = tsplit.Graph(g)
    base = tsplit.Plan.default(G).stats()
    static = base["static_bytes"]
    for frac in (1.0, 0.6, 0.35):
        budget = static + int(frac * (base["peak_extent"] - static))
        P = tsplit.Plan.plan(G, budget)
        st = P.stats()
        assert st["peak_extent"] <= budget
        cfg = P.oracle_cfg()
        ref = sim.simulate(g, cfg)
        assert ref.peak_extent == st["peak_extent"]
        assert [tuple(e) for e in ref.trace] == P.trace()


@pytest.mark.parametrize("kw", [dict(batch=4, hidden=8, depth=2, in_dim=8, classes=3),
                                dict(batch=8, hidden=32, depth=2, in_dim=16, classes=5),
                                dict(batch=4, hidden=64, depth=2, in_dim=64, classes=10)])
def test_t8_planner_feasible_exactly_when_brute_force_is(kw):
    """T8 over a budget sweep on graphs small enough to enumerate every plan (opt x p_num
    per activation, 9^3 plans): the planner reports INFEASIBLE below the brute-force
    optimum (soundness) and finds a plan that fits at every budget from the optimum up
    (on these graphs the heuristic is complete; Alg. 2's choice itself stays unpinned)."""
    g = graphs.mlp(**kw)
    G = tsplit.Graph(g)
    best, _ = brute.min_peak(g, ps=(1, 2, 4))
    top = tsplit.Plan.default(G).stats()["peak_extent"]
    assert best < top
    misses = []
    for budget in range(best - 512, top + 1, 16):
        try:
            P = tsplit.Plan.plan(G, budget)
        except tsplit.TsError as e:
            assert e.status == "ERR_INFEASIBLE"
            if budget >= best:
                misses.append(budget)
            continue
        assert budget >= best, "a plan below the brute-force optimum"
        assert P.stats()["peak_extent"] <= budget
    assert not misses, misses


def test_planner_bert_large_quarter_budget():
    """North-star config: BERT-Large b32 under 25% of the unsplit dynamic peak (R4)."""
    g = graphs.config_graph("bert_large")
    G = tsplit.Graph(g)
    base = tsplit.Plan.default(G).stats()
    static = base["static_bytes"]
    budget = static + (base["peak_extent"] - static) // 4
    P = tsplit.Plan.plan(G, budget)
    st = P.stats()
    assert st["peak_extent"] <= budget
    assert st["n_recompute_tensors"] + st["n_swap_tensors"] > 0


@pytest.mark.parametrize("gname", ["vgg_tiny", "resnet_tiny", "vgg16", "resnet50"])
def test_cnn_schedule_static_and_default_trace(gname):
    g = graphs.config_graph(gname)
    G = tsplit.Graph(g)
    assert G.schedule() == sim.schedule(g)
    assert G.static_bytes() == sim.static_bytes(g)
    if gname.endswith("tiny"):
        _compare(g, sim.default_cfg(g))


@pytest.mark.parametrize("gname,seed", [("vgg_tiny", 0), ("vgg_tiny", 1), ("resnet_tiny", 0), ("resnet_tiny", 1)])
def test_cnn_trace_bit_exact_random_plans(gname, seed):
    g = graphs.config_graph(gname)
    r = random.Random(seed)
    cfg = sim.default_cfg(g)
    for t in brute.act_tensors(g):
        cfg[t] = (r.choice([0, 1, 2]), r.choice([1, 2, 4]), r.choice([1, 2]))
    _compare(g, cfg)


@pytest.mark.parametrize("seed", range(4))
def test_trace_bit_exact_random_plans_bert_tiny_fused_attention(seed):
    """Fused attention (two outputs, one auxiliary): schedule, replays of either
    output, and the allocation trace equal the oracle simulator's."""
    g = graphs.config_graph("bert_tiny", fused_attention=True)
    r = random.Random(100 + seed)
    cfg = sim.default_cfg(g)
    for t in brute.act_tensors(g):
        cfg[t] = (r.choice([0, 1, 2]), r.choice([1, 2, 4]), r.choice([1, 2, 3]))
    _compare(g, cfg)


def test_fused_attention_large_default_and_planned():
    g = graphs.config_graph("bert_large", fused_attention=True)
    G = tsplit.Graph(g)
    st = tsplit.Plan.default(G).stats()
    assert st["peak_extent"] == sim.simulate(g, sim.default_cfg(g)).peak_extent
    P = tsplit.Plan.plan(G, st["static_bytes"] + (st["peak_extent"] - st["static_bytes"]) // 4)
    assert P.stats()["peak_extent"] <= st["static_bytes"] + (st["peak_extent"] - st["static_bytes"]) // 4


@pytest.mark.parametrize("seed", range(6))
def test_trace_bit_exact_lru_recompute_cache(seed):
    """D-LRU: the C++ expansion with a recompute cache limit reproduces the oracle's
    items, replay count and allocation trace bit for bit (bf16 BERT-tiny, random plans)."""
    g = graphs.config_graph("bert_tiny")
    rnd = random.Random(100 + seed)
    acts = brute.act_tensors(g)
    cfg = sim.default_cfg(g)
    for t in acts:
        cfg[t] = (rnd.choice([sim.RESIDE, sim.RECOMPUTE, sim.RECOMPUTE, sim.SWAP]), rnd.choice([1, 1, 2, 4]), 1)
    for cache in (1 << 16, 1 << 20, 2 ** 64 - 1):
        _compare(g, cfg, cache)


def test_planner_lru_cache_feasible_and_not_slower():
    """ts_plan's D-LRU post-pass keeps the plan within the budget and never predicts a
    slower step than the memory-centric plan it starts from; the plan serializes with it."""
    g = graphs.config_graph("bert_large", layers=4)
    G = tsplit.Graph(g)
    st = tsplit.Plan.default(G).stats()
    budget = st["static_bytes"] + int(0.25 * (st["peak_extent"] - st["static_bytes"]))
    P = tsplit.Plan.plan(G, budget)
    s = P.stats()
    assert s["peak_extent"] <= budget
    mc = tsplit.Plan.deserialize(G, P.serialize())
    assert mc.stats()["recompute_cache_bytes"] == s["recompute_cache_bytes"]
    assert mc.trace() == P.trace()
    mc.set_recompute_cache(0)
    assert s["predicted_s"] <= mc.stats()["predicted_s"] + 1e-12
    assert s["n_replay"] <= mc.stats()["n_replay"]


@pytest.mark.parametrize("gname,seed", [("mlp", s) for s in range(6)] + [("bert_tiny", s) for s in range(4)])
def test_trace_bit_exact_channel_split_plans(gname, seed):
    """D-CH channel (parameter-dim) splits: the C++ expansion, pool and trace equal the
    oracle simulator's bit for bit (plans applied with ts_plan_set_many)."""
    from test_oracle_channel import CHAINS, channel_cfg
    g = graphs.config_graph(gname)
    cfg = channel_cfg(g, random.Random(100 + seed), CHAINS[gname], prob=0.9)
    G = tsplit.Graph(g)
    plan = tsplit.Plan.default(G)
    plan.set_many({t: cfg[t] for t in brute.act_tensors(g)})
    ref = sim.simulate(g, cfg)
    got = plan.trace()
    assert len(got) == len(ref.trace)
    for a, b in zip(got, ref.trace):
        assert a == tuple(b), (a, b)
    st = plan.stats()
    assert (st["peak_live"], st["peak_extent"], st["n_replay"]) == (ref.peak_live, ref.peak_extent, ref.n_replay)
    assert [it[0] for it in plan.items()] == [it.kind for it in ref.items]
    for t in brute.act_tensors(g):
        assert plan.get_dim(t) == (sim.dim_of(cfg, t) if cfg[t][1] > 1 else 0)


def test_channel_split_rejected_unless_legal():
    g = graphs.config_graph("bert_tiny")
    names = {t["name"]: t["id"] for t in g["tensors"]}
    plan = tsplit.Plan.default(tsplit.Graph(g))
    before = plan.trace()
    with pytest.raises(tsplit.TsError):   # gelu alone: its input is not channel-split
        plan.set(names["l0.gelu"], 0, 2, 1, dim=1)
    with pytest.raises(tsplit.TsError):   # layernorm output
        plan.set_many({names["l0.ln1"]: (0, 2, 1, 1)})
    assert plan.trace() == before          # unchanged after a rejected call
    plan.set_many({names["l0.ffn1"]: (2, 2, 1, 1), names["l0.gelu"]: (1, 2, 1, 1)})
    assert plan.get_dim(names["l0.ffn1"]) == 1


@pytest.mark.parametrize("frac", [0.8, 0.75])
def test_planner_uses_channel_splits_when_the_batch_is_one(frac):
    """Batch 1 leaves no sample dim to split (Fig. 6), so Alg. 2's split step proposes the
    parameter dim (D-CH) once recomputing one tensor no longer suffices (at 90 % it does):
    the plan fits, splits along dim 1, its trace is the oracle
    simulator's, and executing it gives the unsplit gradients (fp64 oracle)."""
    from oracle import execplan, net
    from tsinputs import gen
    g = graphs.mlp(batch=1, in_dim=64, hidden=2048, depth=3, classes=10)
    G = tsplit.Graph(g)
    st = tsplit.Plan.default(G).stats()
    budget = st["static_bytes"] + int(frac * (st["peak_extent"] - st["static_bytes"]))
    P = tsplit.Plan.plan(G, budget)
    assert P.stats()["peak_extent"] <= budget
    cfg = P.oracle_cfg()
    assert any(c[1] > 1 and c[3] == 1 for c in cfg.values())
    ref = sim.simulate(g, cfg)
    assert P.trace() == [tuple(e) for e in ref.trace]
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    l0, g0, _, _ = net.train_step(g, params, inputs)
    l1, g1 = execplan.execute(g, cfg, params, inputs)
    assert abs(l1 - l0) <= 1e-12 * abs(l0)
    from test_oracle_net_sim import rel_errs
    assert max(rel_errs(g1, g0).values()) <= 1e-12


def test_channel_plan_serialize_roundtrip():
    """A channel-split plan (D-CH) survives ts_plan_serialize / _deserialize (the DP
    broadcast): same per-tensor dims and the same trace."""
    g = graphs.config_graph("bert_tiny")
    names = {t["name"]: t["id"] for t in g["tensors"]}
    G = tsplit.Graph(g)
    P = tsplit.Plan.default(G)
    P.set_many({names["l0.ffn1"]: (2, 4, 1, 1), names["l0.gelu"]: (1, 4, 3, 1), names["l1.q"]: (2, 2, 1, 0)})
    Q = tsplit.Plan.deserialize(G, P.serialize())
    assert Q.trace() == P.trace()
    for t in brute.act_tensors(g):
        assert (Q.get(t), Q.get_dim(t)) == (P.get(t), P.get_dim(t))


def test_plan_deserialize_rejects_bad_blobs():
    """ts_plan_deserialize validates like ts_plan_set: a blob of another graph (fingerprint),
    a truncated one, p = 0 / 3, a swapped parameter — TS_ERR_ARG, nothing adopted."""
    import struct
    g = graphs.config_graph("bert_tiny")
    G = tsplit.Graph(g)
    blob = bytearray(tsplit.Plan.default(G).serialize())
    tsplit.Plan.deserialize(G, bytes(blob))  # the round trip itself is fine
    other = tsplit.Graph(graphs.config_graph("bert_tiny", hidden=256, heads=4))
    with pytest.raises(tsplit.TsError):
        tsplit.Plan.deserialize(other, bytes(blob))
    g2 = tsplit.Graph(graphs.config_graph("bert_tiny", batch=8))  # same tensor count, other shapes
    with pytest.raises(tsplit.TsError):
        tsplit.Plan.deserialize(g2, bytes(blob))
    with pytest.raises(tsplit.TsError):
        tsplit.Plan.deserialize(G, bytes(blob[:-12]))
    act = brute.act_tensors(g)[0]
    param = next(t["id"] for t in g["tensors"] if t["kind"] == "param")
    for tid, word, value in ((act, 1, 0), (act, 1, 3), (param, 0, tsplit.SWAP), (act, 4, 3)):  # (a lag needs swap)
        bad = bytearray(blob)
        struct.pack_into("<i", bad, 24 + 20 * tid + 4 * word, value)
        with pytest.raises(tsplit.TsError):
            tsplit.Plan.deserialize(G, bytes(bad))


def test_plan_roofline_bounds():
    """ts_plan_roofline: sum over micro-ops of max(F / P, bytes / BW) — at least each of the
    two totals' own bound, at most their sum; its FLOP equal the plan's compute FLOP (recompute
    replays included); splitting changes no algorithmic FLOP."""
    g = graphs.config_graph("bert_tiny")
    G = tsplit.Graph(g)
    P0 = tsplit.Plan.default(G)
    pk, bw = 1.4e15, 6.5e12
    s, f, b = P0.roofline(pk, bw)
    assert max(f / pk, b / bw) <= s <= f / pk + b / bw
    assert f == pytest.approx(P0.stats()["compute_flop"], rel=1e-12)
    P1 = tsplit.Plan.default(G)
    names = G.names
    P1.set(names["l0.ffn1"], tsplit.RESIDE, 4, 1)
    P1.set(names["l1.q"], tsplit.RECOMPUTE, 1, 1)
    s1, f1, b1 = P1.roofline(pk, bw)
    assert f1 == pytest.approx(P1.stats()["compute_flop"], rel=1e-12) and f1 > f


@pytest.mark.parametrize("gname,seed", [("vgg_tiny", 0), ("vgg_tiny", 1), ("resnet_tiny", 0), ("resnet_tiny", 1),
                                        ("vgg16", 2), ("resnet50", 3)])
def test_trace_bit_exact_band_split_plans(gname, seed):
    """D-ATTR attribute (height) splits: the C++ expansion, staging temporaries, pool and
    trace equal the oracle simulator's bit for bit."""
    from test_oracle_attr import _rand_attr_cfg
    over = {"batch": 4} if gname in ("vgg16", "resnet50") else {}
    g = graphs.config_graph(gname, **over)
    cfg = _rand_attr_cfg(g, random.Random(200 + seed))
    for t in brute.act_tensors(g):   # random D-LAG lags on swapped tensors
        if cfg[t][0] == sim.SWAP and seed % 2:
            cfg[t] = cfg[t][:3] + ((cfg[t][3] if len(cfg[t]) > 3 else 0), 2)
    G = tsplit.Graph(g)
    plan = tsplit.Plan.default(G)
    plan.set_many({t: cfg[t] for t in brute.act_tensors(g)})
    ref = sim.simulate(g, cfg)
    got = plan.trace()
    assert any(k >= 2 * len(g["tensors"]) for _, _, _, k, _, _, _ in got)   # staging temporaries present
    assert len(got) == len(ref.trace)
    for a, b in zip(got, ref.trace):
        assert a == tuple(b), (a, b)
    st = plan.stats()
    assert (st["peak_live"], st["peak_extent"], st["n_replay"]) == (ref.peak_live, ref.peak_extent, ref.n_replay)
    assert [it[0] for it in plan.items()] == [it.kind for it in ref.items]
    for t in brute.act_tensors(g):
        assert plan.get_dim(t) == (sim.dim_of(cfg, t) if cfg[t][1] > 1 else 0)


def test_band_split_rejected_unless_legal():
    g = graphs.config_graph("vgg_tiny")
    names = {t["name"]: t["id"] for t in g["tensors"]}
    plan = tsplit.Plan.default(tsplit.Graph(g))
    with pytest.raises(tsplit.TsError):   # relu0 must follow conv0's band split
        plan.set(names["conv0"], tsplit.RESIDE, 2, 1, dim=2)
    plan.set_many({names["conv0"]: (0, 2, 1, 2), names["relu0"]: (0, 2, 1, 2)})
    with pytest.raises(tsplit.TsError):   # a 2-D tensor has no height
        plan.set(names["fc0"], tsplit.RESIDE, 2, 1, dim=2)
    last = [t for t in g["tensors"] if t["kind"] == "act" and len(t["shape"]) == 4][-1]
    with pytest.raises(tsplit.TsError):   # read by flatten
        plan.set(last["id"], tsplit.RESIDE, 2, 1, dim=2)


def test_planner_uses_band_splits_when_the_batch_is_one():
    """Batch 1 (Fig. 6): with no sample dim Alg. 2's split step proposes the height
    (D-ATTR).  VGG at half its dynamic peak is infeasible without splits and feasible with
    bands; the plan's trace is the simulator's and executing it (fp64 oracle) gives the
    unsplit gradients."""
    from oracle import execplan, net
    from tsinputs import gen
    from test_oracle_net_sim import rel_errs
    g = graphs.config_graph("vgg_small", batch=1, dtype="f32")
    G = tsplit.Graph(g)
    st = tsplit.Plan.default(G).stats()
    budget = st["static_bytes"] + int(0.5 * (st["peak_extent"] - st["static_bytes"]))
    with pytest.raises(tsplit.TsError):
        tsplit.Plan.plan(G, budget, no_split=True)
    P = tsplit.Plan.plan(G, budget)
    assert P.stats()["peak_extent"] <= budget
    cfg = P.oracle_cfg()
    assert any(c[1] > 1 and len(c) > 3 and c[3] == 2 for c in cfg.values())
    assert P.trace() == [tuple(e) for e in sim.simulate(g, cfg).trace]
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    l0, g0, _, _ = net.train_step(g, params, inputs)
    l1, g1 = execplan.execute(g, cfg, params, inputs)
    assert abs(l1 - l0) <= 1e-12 * abs(l0)
    assert max(rel_errs(g1, g0).values()) <= 1e-12


def test_band_plan_serialize_roundtrip():
    g = graphs.config_graph("vgg_small", batch=1)
    G = tsplit.Graph(g)
    st = tsplit.Plan.default(G).stats()
    P = tsplit.Plan.plan(G, st["static_bytes"] + int(0.5 * (st["peak_extent"] - st["static_bytes"])))
    Q = tsplit.Plan.deserialize(G, P.serialize())
    assert Q.trace() == P.trace() and Q.oracle_cfg() == P.oracle_cfg()


@pytest.mark.parametrize("gname,seed", [("vgg_tiny", 0), ("vgg_tiny", 1), ("resnet_tiny", 0), ("resnet_tiny", 1),
                                        ("vgg16", 2), ("resnet50", 3)])
def test_trace_bit_exact_channel4_plans(gname, seed):
    """D-CH on NHWC images (conv / BN / pool / add channel blocks, staged merges): the C++
    expansion and trace equal the oracle simulator's bit for bit."""
    from test_oracle_channel4 import rand_chan4_cfg
    over = {"batch": 4} if gname in ("vgg16", "resnet50") else {}
    g = graphs.config_graph(gname, **over)
    cfg = rand_chan4_cfg(g, random.Random(500 + seed))
    plan = tsplit.Plan.default(tsplit.Graph(g))
    plan.set_many({t: cfg[t] for t in brute.act_tensors(g)})
    ref = sim.simulate(g, cfg)
    got = plan.trace()
    assert len(got) == len(ref.trace)
    for a, b in zip(got, ref.trace):
        assert a == tuple(b), (a, b)
    assert [it[0] for it in plan.items()] == [it.kind for it in ref.items]
    for t in brute.act_tensors(g):
        assert plan.get_dim(t) == (sim.dim_of(cfg, t) if cfg[t][1] > 1 else 0)
