"""Channel (parameter-dim) splits, reading D-CH (Fig. 6): the oracle's
expansion and piece-by-piece execution with activations split into column blocks.
Pinned by T1 (any plan = the unsplit gradients, fp64) and by the legality rules."""
import random

import pytest

from oracle import brute, execplan, net, sim
from tsinputs import gen, graphs

from test_oracle_net_sim import rel_errs

CHAINS = {"mlp": [("fc0", "relu0"), ("fc1", "relu1")],
          "bert_tiny": [("l0.ffn1", "l0.gelu"), ("l1.ffn1", "l1.gelu")]}


def channel_cfg(g, r, chains, ps=(2, 4), prob=0.8):
    """Random sample-dim plan, then channel-split (dim 1) linear -> elementwise chains with
    random options; the chains' neighbours are made legal (unsplit)."""
    names = {t["name"]: t["id"] for t in g["tensors"]}
    ops_by_out = {o["outputs"][0]: o for o in g["ops"]}
    cfg = sim.default_cfg(g)
    for t in brute.act_tensors(g):
        cfg[t] = (r.choice([0, 1, 2]), r.choice([p for p in (1, 2, 4) if g["samples"] % p == 0]), r.choice([1, 2, 3]))
    chosen = []
    for chain in chains:
        if r.random() < prob:
            p = r.choice(ps)
            for nm in chain:
                cfg[names[nm]] = (r.choice([0, 1, 2]), p, r.choice([1, 2]), 1)
            chosen.append(chain)
    consumers = {}
    for o in g["ops"]:
        for t in o["inputs"]:
            consumers.setdefault(t, []).append(o)
    for chain in chosen:
        lin = ops_by_out[names[chain[0]]]
        x = lin["inputs"][0]
        if g["tensors"][x]["kind"] == "act" and sim.dim_of(cfg, x) != 1:
            cfg[x] = (cfg[x][0], 1, cfg[x][2])
        for c in consumers[names[chain[-1]]]:
            y = c["outputs"][0]
            if c["kind"] == "linear" and sim.dim_of(cfg, y) != 1 and g["tensors"][y]["kind"] == "act":
                cfg[y] = (cfg[y][0], 1, cfg[y][2])
    sim.check_channel(g, cfg)
    return cfg


@pytest.mark.parametrize("gname", ["mlp", "bert_tiny"])
def test_t1_channel_split_plans_same_gradients(gname):
    g = graphs.config_graph(gname)
    P, I = gen.init_params(g), gen.make_inputs(g)
    loss, pg, _, _ = net.train_step(g, P, I)
    r = random.Random(11)
    for _ in range(10 if gname == "mlp" else 4):
        cfg = channel_cfg(g, r, CHAINS[gname])
        l2, pg2 = execplan.execute(g, cfg, P, I)
        assert abs(l2 - loss) <= 1e-12 * abs(loss)
        errs = rel_errs(pg2, pg)
        assert max(errs.values()) <= 1e-12, max(errs.items(), key=lambda kv: kv[1])


def test_channel_micro_ops_and_pieces():
    """fc0 -> relu0 split into 4 column blocks: 4 channel micro-ops each, every piece a
    quarter of the tensor; fc1 (sample mode) reads all four blocks of relu0."""
    g = graphs.mlp()
    names = {t["name"]: t["id"] for t in g["tensors"]}
    cfg = sim.default_cfg(g)
    cfg[names["fc0"]] = (sim.RESIDE, 4, 1, 1)
    cfg[names["relu0"]] = (sim.SWAP, 4, 1, 1)
    items, _, _, fwd_end, an = sim.expand(g, cfg)
    f = [it for it in items[:fwd_end]]
    fc0 = [it for it in f if g["ops"][it.op]["name"] == "fc0"]
    relu0 = [it for it in f if g["ops"][it.op]["name"] == "relu0"]
    fc1 = [it for it in f if g["ops"][it.op]["name"] == "fc1"]
    assert [it.writes for it in fc0] == [[(names["fc0"], k)] for k in range(4)]
    assert [it.reads for it in relu0] == [[(names["fc0"], k)] for k in range(4)]
    assert len(fc1) == 1 and sorted(fc1[0].reads) == [(names["relu0"], j) for j in range(4)]
    r = sim.simulate(g, cfg)
    quarter = an.bytes_[names["relu0"]] // 4
    assert r.d2h_bytes == r.h2d_bytes == 4 * quarter  # every block swapped out and back
    # the backward of fc1 (sample mode) writes the gradient of every block of relu0
    b_fc1 = next(it for it in items if it.kind == "B" and g["ops"][it.op]["name"] == "fc1")
    n = an.n
    assert sorted(w for w in b_fc1.writes if w[0] == n + names["relu0"]) == [(n + names["relu0"], j) for j in range(4)]


@pytest.mark.parametrize("bad", ["ln_producer", "mismatched_p", "dropout_consumer"])
def test_channel_split_legality(bad):
    g = graphs.config_graph("bert_tiny")
    names = {t["name"]: t["id"] for t in g["tensors"]}
    cfg = sim.default_cfg(g)
    if bad == "ln_producer":      # a layernorm cannot write column blocks
        cfg[names["l0.ln1"]] = (0, 2, 1, 1)
    elif bad == "mismatched_p":   # gelu's input and output blocks must match
        cfg[names["l0.ffn1"]] = (0, 2, 1, 1)
        cfg[names["l0.gelu"]] = (0, 4, 1, 1)
    else:                         # the q projection feeds the (unfused) attention scores
        cfg[names["l0.q"]] = (0, 2, 1, 1)
    with pytest.raises(ValueError):
        sim.check_channel(g, cfg)
