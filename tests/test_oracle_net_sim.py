"""Pins of oracle/net.py, oracle/sim.py, oracle/execplan.py, oracle/brute.py and
oracle/cost.py."""

import random

import numpy as np
import pytest

from conftest import rel_errs
from oracle import brute, cost, execplan, net, sim
from tsinputs import gen, graphs

MB = 1e6


# ----------------------------------------------------------------------------- net
def _fd_param(graph, params, inputs, name, n=3, h=1e-6, seed=0):
    loss, pg, _, _ = net.train_step(graph, params, inputs)
    r = np.random.default_rng(seed)
    for _ in range(n):
        d = r.standard_normal(params[name].shape)
        p1 = dict(params); p1[name] = params[name].astype(np.float64) + h * d
        p2 = dict(params); p2[name] = params[name].astype(np.float64) - h * d
        num = (net.train_step(graph, p1, inputs)[0] - net.train_step(graph, p2, inputs)[0]) / (2 * h)
        ana = float(np.sum(pg[name] * d))
        assert abs(num - ana) <= 1e-6 * max(abs(ana), 1e-3), (name, num, ana)


def test_mlp_whole_net_fd():
    g = graphs.mlp()
    P, I = gen.init_params(g), gen.make_inputs(g)
    for name in ["fc0.w", "fc1.b", "fc2.w"]:
        _fd_param(g, P, I, name)


def test_bert_tiny_whole_net_fd():
    g = graphs.config_graph("bert_tiny", layers=1, hidden=32, heads=2, seq=8, batch=2, vocab=40)
    P, I = gen.init_params(g), gen.make_inputs(g)
    for name in ["emb.word", "emb.pos", "l0.q.w", "l0.ln1.g", "l0.ffn1.b", "pool.w", "cls.w"]:
        _fd_param(g, P, I, name, n=2)


# ----------------------------------------------------------------------- schedule
def _dag(edges, n):
    """Tiny DFG whose op i consumes the outputs of ops in edges[i]."""
    b = graphs.GraphBuilder("dag", "f32", 1)
    x = b.tensor("x", (1, 1), "input")
    outs = {}
    for i in range(n):
        ins = [outs[j] for j in edges.get(i, [])] or [x]
        outs[i] = b.op("add" if len(ins) == 2 else "relu", f"o{i}", ins[:2], (1, 1))
    return b.done()


def test_alg1_dfs_order_hand_worked():
    # A->B, A->C, B->D, D->E, C->E: DFS manner visits B's subtree before C
    g = _dag({1: [0], 2: [0], 3: [1], 4: [3, 2]}, 5)
    assert sim.schedule(g) == [0, 1, 3, 2, 4]
    # diamond: E becomes ready only after both branches
    g = _dag({1: [0], 2: [0], 3: [1, 2]}, 4)
    assert sim.schedule(g) == [0, 1, 2, 3]


def test_alg1_is_topological_on_bert():
    g = graphs.config_graph("bert_tiny")
    order = sim.schedule(g)
    pos = {o: i for i, o in enumerate(order)}
    prod = {o["outputs"][0]: o["id"] for o in g["ops"]}
    for o in g["ops"]:
        for t in o["inputs"]:
            if t in prod:
                assert pos[prod[t]] < pos[o["id"]]
    assert sorted(order) == list(range(len(g["ops"])))


# ------------------------------------------------------------------ T2 Table II
def test_table2_tensor_size_distribution():
    """PAPER.md Table II (L85-112): BERT-Large fp32, b32 s512 a16."""
    g = graphs.bert(dtype="f32")
    counts = [0] * 6
    edges = [1, 10, 50, 100, 500]
    for t in g["tensors"]:
        mb = graphs.tensor_bytes(t) / MB
        counts[sum(mb >= e for e in edges)] += 1
    assert counts[1:] == [98, 48, 243, 49, 72]
    # with the paper's 27 tensors below 1 MB the printed percentages reproduce
    total = 27 + sum(counts[1:])
    pct = [round(100 * c / total, 2) for c in [27] + counts[1:]]
    assert pct == [5.03, 18.25, 8.94, 45.25, 9.12, 13.41]


# ------------------------------------------------------------------- T3 worked example
def test_t3_worked_example_memory_sets():
    """M_0 = {X, W1, W2}; M_1 = M_0 + {s1}; at dConv2 (N-2):
    {X, W1, W2, s1, s3, s'1, s'2, W'2}.  Conv layers are modelled as linear ops
    (the memory model is op-agnostic); s3 is read as the loss output (G10)."""
    b = graphs.GraphBuilder("t3", "f32", 4)
    X = b.tensor("X", (4, 8), "input")
    Y = b.tensor("labels", (4,), "label", dtype="i32")
    W1 = b.param("W1", (8, 8)); b1 = b.param("b1", (8,))
    W2 = b.param("W2", (3, 8)); b2 = b.param("b2", (3,))
    s1 = b.op("linear", "conv1", [X, W1, b1], (4, 8))
    s2 = b.op("linear", "conv2", [s1, W2, b2], (4, 3))
    s3 = b.op("xent", "loss", [s2, Y], (1,), out_dtype="f32")
    g = b.done()
    r = sim.simulate(g)
    n = len(g["tensors"])
    live = set()
    sets = []
    ev = {}
    for seq, item, kind, key, j, off, nb in r.trace:
        ev.setdefault(item, []).append((kind, key))
    for e in ev.get(-1, []):
        live.add(e[1])
    for i, it in enumerate(r.items):
        for kind, key in ev.get(i, []):
            if kind == "A":
                live.add(key)
        sets.append((it.kind, set(live)))
        for kind, key in ev.get(i, []):
            if kind == "F":
                live.discard(key)
    names = lambda s: {("d" + g["tensors"][k - n]["name"]) if k >= n else g["tensors"][k]["name"] for k in s}
    # params are static (always live); labels are an input the paper's figure omits
    assert [k for k, _ in sets] == ["F", "F", "F", "B", "B", "B"]
    assert names(sets[0][1]) - {"labels"} == {"X", "conv1"}                      # M_1 (+ params)
    m_n2 = names(sets[4][1]) - {"labels"}                                        # dConv2
    assert m_n2 == {"X", "conv1", "loss", "dconv1", "dconv2"}                    # + W1, W2, W'2 static
    assert "conv2" not in m_n2


# ------------------------------------------------------------------- T1 invariance
def _rand_cfg(g, r, ps=(1, 2, 4)):
    cfg = sim.default_cfg(g)
    for t in brute.act_tensors(g):
        cfg[t] = (r.choice([0, 1, 2]), r.choice([p for p in ps if g["samples"] % p == 0]), r.choice([1, 2, 3]))
    return cfg


@pytest.mark.parametrize("gname", ["mlp", "bert_tiny"])
def test_t1_any_plan_same_gradients(gname):
    g = graphs.config_graph(gname)
    P, I = gen.init_params(g), gen.make_inputs(g)
    loss, pg, _, _ = net.train_step(g, P, I)
    r = random.Random(3)
    for trial in range(4 if gname == "bert_tiny" else 12):
        cfg = _rand_cfg(g, r)
        l2, pg2 = execplan.execute(g, cfg, P, I)
        assert abs(l2 - loss) <= 1e-12 * abs(loss)
        errs = rel_errs(pg2, pg)
        assert max(errs.values()) <= 1e-12, max(errs.items(), key=lambda kv: kv[1])


# ------------------------------------------------------------------ T5 recompute
@pytest.mark.parametrize("N", [1, 2, 3, 5, 8])
def test_t5_memory_centric_recompute_count(N):
    """P:L294 Fig. 11: a chain op1..opN with only op1's input checkpointed runs
    N(N+1)/2 extra operations."""
    b = graphs.GraphBuilder("chain", "f32", 2)
    X = b.tensor("X", (2, 4), "input")
    Y = b.tensor("labels", (2,), "label", dtype="i32")
    W = b.param("W", (4, 4)); bb = b.param("b", (4,))
    a = b.op("linear", "op1", [X, W, bb], (2, 4))
    acts = [a]
    for i in range(2, N + 1):
        a = b.op("gelu", f"op{i}", [a], (2, 4))
        acts.append(a)
    b.op("xent", "loss", [a, Y], (1,), out_dtype="f32")
    g = b.done()
    cfg = sim.default_cfg(g)
    for t in acts:
        cfg[t] = (sim.RECOMPUTE, 1, 1)
    r = sim.simulate(g, cfg)
    assert r.n_replay == N * (N + 1) // 2
    # and the peak never holds more than one recomputed chain tensor beyond the
    # working set (O(1) memory): fewer live pieces than the all-reside plan
    assert r.peak_live <= sim.simulate(g).peak_live
    P, I = gen.init_params(g), gen.make_inputs(g)
    l0, g0, _, _ = net.train_step(g, P, I)
    l1, g1 = execplan.execute(g, cfg, P, I)
    assert max(rel_errs(g1, g0).values()) <= 1e-12


# -------------------------------------------------------------- T6 in-place re-split
def test_t6_resplit_2_to_4_is_in_place():
    g = graphs.mlp()
    cfg = sim.default_cfg(g)
    names = {t["name"]: t["id"] for t in g["tensors"]}
    cfg[names["fc0"]] = (sim.RESIDE, 2, 1)
    cfg[names["relu0"]] = (sim.RESIDE, 4, 1)
    r = sim.simulate(g, cfg)
    relu_items = [i for i, it in enumerate(r.items) if it.kind == "F" and g["ops"][it.op]["name"] == "relu0"]
    assert len(relu_items) == 4
    # the 4 micro-ops read pieces 0,0,1,1 of the 2-way input: no allocation or copy of fc0
    reads = [r.items[i].reads[0] for i in relu_items]
    assert [j for _, j in reads] == [0, 0, 1, 1]
    allocs = [(e[3], e[1]) for e in r.trace if e[2] == "A" and e[1] in relu_items]
    assert all(key != names["fc0"] for key, _ in allocs)
    assert not any(it.kind in ("SO", "SI") for it in r.items)


# ------------------------------------------------------------------ T7 Eq. 3
def test_t7_eq3_special_cases():
    S, B = 1e9, 5e10
    T = [1e-3] * 10
    # no overlap window, link idle: the full transfer both ways is exposed
    assert cost.eq3_swap_cost(S, B, B, T, [0.0] * 10, 3, 4, 6, 6) == pytest.approx(2 * S / B)
    # windows longer than S/B: fully hidden
    T2 = [1.0] * 10
    assert cost.eq3_swap_cost(S, B, B, T2, [0.0] * 10, 0, 9, 2, 9) == 0.0
    # a busy link (Oc = 1) gives no window at all
    assert cost.eq3_swap_cost(S, B, B, T2, [1.0] * 10, 0, 9, 2, 9) == pytest.approx(2 * S / B)


def test_eq2_delta_m_is_the_size_by_simulation():
    """Eq. 2: swapping or recomputing a tensor that is live across op i but
    not touched by it lowers the memory requirement at op i by exactly size(s_j) (256-B
    aligned pieces) — checked against the simulator's live bytes, not restated."""
    g = graphs.mlp()
    names = {t["name"]: t["id"] for t in g["tensors"]}
    base = sim.simulate(g)
    t = names["relu0"]  # held for fc1's backward, not read by relu1 / fc2 / loss forward
    for opt in (sim.SWAP, sim.RECOMPUTE):
        cfg = sim.default_cfg(g)
        cfg[t] = (opt, 1, 1)
        if opt == sim.RECOMPUTE:  # the replay's input fc0 is recomputed too (else it is held instead)
            cfg[names["fc0"]] = (sim.RECOMPUTE, 1, 1)
        r = sim.simulate(g, cfg)
        for op_name in ("relu1", "fc2", "loss"):
            i0 = next(i for i, it in enumerate(base.items) if it.kind == "F" and g["ops"][it.op]["name"] == op_name)
            i1 = next(i for i, it in enumerate(r.items) if it.kind == "F" and g["ops"][it.op]["name"] == op_name)
            dm = base.live_after_alloc[i0] - r.live_after_alloc[i1]
            assert dm == sim.align(cost.eq2_delta_m(sim.tbytes(g["tensors"][t]))), (opt, op_name, dm)


def test_eq6_split_term_equals_the_planner_timeline():
    """Eq. 6 (reading R7) with c = reside: the cost of splitting is the
    dT_split term alone, sum_k T(op on split k) - T(op), over every op whose micro-op count
    changes.  The C++ planner's predicted step time (D-TIME timeline over the analytic
    profile) must move by exactly that when a tensor is split 2 or 4 ways."""
    from paper_conf_icde_niemyc22_b200 import tsplit
    g = graphs.mlp()
    G = tsplit.Graph(g)
    prof = tsplit.Profile(G)
    base = tsplit.Plan.default(G).stats()["predicted_s"]
    names = {t["name"]: t["id"] for t in g["tensors"]}
    for name, p in (("relu0", 2), ("fc1", 4), ("relu1", 2)):
        t = names[name]
        P = tsplit.Plan.default(G)
        P.set(t, tsplit.RESIDE, p, 1)
        got = P.stats()["predicted_s"] - base
        touched = [o for o, op in enumerate(g["ops"]) if t in op["inputs"] + op["outputs"]]
        want = sum(cost.eq6_split_cost(p, 0.0, sum(prof.get(o, p)), sum(prof.get(o, 1))) for o in touched)
        assert got == pytest.approx(want, rel=1e-9, abs=1e-15), (name, got, want)


# ------------------------------------------------------------ T9 brute force
def _tiny():
    return graphs.mlp(batch=4, hidden=8, depth=2, in_dim=8, classes=3)


def test_t9_peak_equals_independent_live_sum_all_plans():
    g = _tiny()
    count = 0
    for cfg in brute.enumerate_plans(g, ps=(1, 2, 4)):
        r = sim.simulate(g, cfg)
        assert r.peak_live == brute.independent_peak(r)
        assert r.peak_extent >= r.peak_live
        count += 1
    assert count == 9 ** 3


def test_t9_equal_sizes_extent_equals_live():
    # all dynamic pieces of one size: best fit never fragments
    b = graphs.GraphBuilder("eq", "f32", 4)
    X = b.tensor("X", (4, 64), "input")
    a = X
    for i in range(4):
        a = b.op("relu", f"r{i}", [a], (4, 64))
    g = b.done()
    r = sim.simulate(g)
    assert r.peak_extent == r.peak_live


def test_t8_infeasible_budget_has_no_plan():
    g = _tiny()
    best, _ = brute.min_peak(g, ps=(1, 2, 4))
    assert best > sim.static_bytes(g)
    for cfg in brute.enumerate_plans(g, ps=(1, 2, 4)):
        assert sim.simulate(g, cfg).peak_extent >= best


def test_pool_best_fit_and_tail_rule():
    p = sim.Pool(0, 4096)
    a = p.alloc(256); b_ = p.alloc(512); c = p.alloc(256); d = p.alloc(256)
    p.release(a, 256); p.release(c, 256)
    # two 256 holes (0 and 768) and the tail: lowest offset hole wins the tie
    assert p.alloc(200) == 0
    # a 512 request fits no hole -> tail
    assert p.alloc(512) == 1280
    p.release(b_, 512)
    # holes: 256@256? no - b_ at 256..768 merged with hole at 768..1024 -> 768 bytes at 256
    assert p.free[0] == (256, 768)
    # best fit prefers the smaller adequate hole over the tail even if the tail is smaller
    q = sim.Pool(0, 1024)
    x = q.alloc(512); y = q.alloc(256)
    q.release(x, 512)           # hole 512 at 0, tail 256 at 768
    assert q.alloc(200) == 0    # tail is used only when nothing else fits


# ------------------------------------------------------------- D-LRU recompute cache
def _chain(N):
    b = graphs.GraphBuilder("chain", "f32", 2)
    X = b.tensor("X", (2, 4), "input")
    Y = b.tensor("labels", (2,), "label", dtype="i32")
    W = b.param("W", (4, 4)); bb = b.param("b", (4,))
    a = b.op("linear", "op1", [X, W, bb], (2, 4))
    acts = [a]
    for i in range(2, N + 1):
        a = b.op("gelu", f"op{i}", [a], (2, 4))
        acts.append(a)
    b.op("xent", "loss", [a, Y], (1,), out_dtype="f32")
    g = b.done()
    cfg = sim.default_cfg(g)
    for t in acts:
        cfg[t] = (sim.RECOMPUTE, 1, 1)
    return g, cfg


@pytest.mark.parametrize("N", [1, 2, 3, 5, 8])
def test_lru_recompute_counts_on_the_fig11_chain(N):
    """the speed-centric strategy recomputes the N ancestors once (O(N)); the
    memory-centric one N(N+1)/2 times; the LRU hybrid keeps the most recently used
    regenerated tensors up to the memory limit.  On the chain, backward group i needs
    op_{N-i}'s output: with room for K regenerated tensors (K >= 2) every miss replays
    the chain up to the needed tensor and the K - 1 tensors before it stay for the next
    K - 1 groups, so the replays are N + (N - K) + (N - 2K) + ...; with K = 1 the one kept
    tensor is always the one just consumed, i.e. memory-centric again."""
    g, cfg = _chain(N)
    piece = 2 * 4 * 4  # one [2, 4] fp32 activation
    assert sim.simulate(g, cfg, cache_bytes=0).n_replay == N * (N + 1) // 2
    assert sim.simulate(g, cfg, cache_bytes=piece).n_replay == N * (N + 1) // 2
    assert sim.simulate(g, cfg, cache_bytes=2 ** 64 - 1).n_replay == N
    for K in (2, 3):
        want = sum(N - K * i for i in range(N) if N - K * i >= 1)
        assert sim.simulate(g, cfg, cache_bytes=K * piece).n_replay == want
    # caching trades memory for replays: the unbounded cache holds the whole chain at once
    if N >= 3:
        assert sim.simulate(g, cfg, cache_bytes=2 ** 64 - 1).peak_live > sim.simulate(g, cfg).peak_live


@pytest.mark.parametrize("seed", range(4))
def test_t1_lru_plans_compute_the_unsplit_gradients(seed):
    """T1 with the recompute cache: any plan and any cache limit give the unsplit
    gradients (fp64, 1e-12), and the simulator finds every read resident."""
    g = graphs.mlp(batch=4, hidden=8, depth=3, in_dim=8, classes=3)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    ref_loss, ref_g, _, _ = net.train_step(g, params, inputs)
    rnd = random.Random(seed)
    acts = brute.act_tensors(g)
    for _ in range(4):
        cfg = sim.default_cfg(g)
        for t in acts:
            cfg[t] = (rnd.choice([sim.RESIDE, sim.RECOMPUTE, sim.RECOMPUTE, sim.SWAP]), rnd.choice([1, 2, 4]), 1)
        cache = rnd.choice([0, 64, 256, 1024, 2 ** 64 - 1])
        loss, grads = execplan.execute(g, cfg, params, inputs, cache_bytes=cache)
        sim.simulate(g, cfg, cache_bytes=cache)
        assert abs(loss - ref_loss) <= 1e-12 * abs(ref_loss)
        assert max(rel_errs(grads, ref_g).values()) <= 1e-12
