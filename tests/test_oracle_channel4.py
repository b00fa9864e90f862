"""Channel (parameter-dim) splits of NHWC activations, reading D-CH (4-D part):
conv2d in channel mode (weight rows / bias block k), channel-local ReLU / add / batch norm /
max pooling, and a conv reading every block through a staged merge (Fig. 6).
T1 invariance in fp64 over random plans mixing channel and sample splits with swap and
recompute, and the legality rules."""

import random

import pytest

from conftest import rel_errs
from oracle import execplan, net, sim
from tsinputs import gen, graphs


def chan_components(g):
    """Groups of 4-D activations joined by channel-local ops (they share one channel split)."""
    ts, ops = g["tensors"], g["ops"]
    parent = {t["id"]: t["id"] for t in ts if t["kind"] == "act" and len(t["shape"]) == 4}

    def find(a):
        while parent[a] != a:
            a = parent[a]
        return a
    for o in ops:
        if o["kind"] in sim.CHANNEL_LOCAL4:
            for x in o["inputs"]:
                if x in parent and o["outputs"][0] in parent:
                    parent[find(x)] = find(o["outputs"][0])
    comp = {}
    for t in parent:
        comp.setdefault(find(t), []).append(t)
    return list(comp.values())


def rand_chan4_cfg(g, r, ps=(2, 4), min_block=1):
    """Random legal plan with NHWC channel splits: options at random, then each channel group
    in turn takes a channel split (C / p >= min_block, a multiple of it), a sample split or
    none, when legal."""
    ts = g["tensors"]
    acts = [t["id"] for t in ts if t["kind"] == "act" and t["name"] != "loss"]
    for _ in range(20):
        cfg = {t["id"]: (0, 1, 1) for t in ts}
        for t in acts:
            cfg[t] = (r.choice([0, 1, 2]), 1, 1)
        comps = chan_components(g)
        r.shuffle(comps)
        for comp in comps:
            mode = r.choice(["chan", "chan", "sample", "none"])
            p = r.choice(ps)
            if mode == "chan" and any((ts[t]["shape"][-1] // p) % min_block or ts[t]["shape"][-1] % p for t in comp):
                continue
            trial = dict(cfg)
            for t in comp:
                opt = cfg[t][0]
                trial[t] = (opt, p, 1, 1) if mode == "chan" else (opt, p, 1, 0) if mode == "sample" else (opt, 1, 1)
            try:
                sim.expand(g, trial)
                cfg = trial
            except ValueError:
                pass
        if any(sim.dim_of(cfg, t) == 1 and cfg[t][1] > 1 and len(ts[t]["shape"]) == 4 for t in acts):
            return cfg
    raise AssertionError("no channel split drawn")


@pytest.mark.parametrize("gname,seed", [("vgg_tiny", 0), ("vgg_tiny", 1), ("resnet_tiny", 0), ("resnet_tiny", 1),
                                        ("resnet_tiny", 2)])
def test_t1_channel4_plans_compute_the_unsplit_gradients(gname, seed):
    g = graphs.config_graph(gname, dtype="f32")
    P, I = gen.init_params(g), gen.make_inputs(g)
    loss, pg, _, _ = net.train_step(g, P, I)
    r = random.Random(seed)
    for trial in range(2):
        cfg = rand_chan4_cfg(g, r)
        l2, pg2 = execplan.execute(g, cfg, P, I, cache_bytes=r.choice([0, 1 << 20]))
        assert abs(l2 - loss) <= 1e-12 * abs(loss)
        assert max(rel_errs(pg2, pg).values()) <= 1e-12


def test_channel4_legality():
    g = graphs.config_graph("vgg_tiny", dtype="f32")
    ts = g["tensors"]
    nm = {t["name"]: t["id"] for t in ts}
    base = {t["id"]: (0, 1, 1) for t in ts}
    cfg = dict(base)
    cfg[nm["conv0"]] = (0, 2, 1, 1)   # relu0 must follow
    with pytest.raises(ValueError):
        sim.expand(g, cfg)
    cfg[nm["relu0"]] = (0, 2, 1, 1)   # pool1 is channel-local: must follow too
    with pytest.raises(ValueError):
        sim.expand(g, cfg)
    cfg[nm["pool1"]] = (0, 2, 1, 1)
    sim.expand(g, cfg)                # conv1 reads the blocks through a staged merge
    bad = dict(cfg)
    bad[nm["conv1"]] = (0, 2, 1, 1)   # a channel-split conv output needs an unsplit input
    with pytest.raises(ValueError):
        sim.expand(g, bad)
    bad = dict(cfg)
    bad[nm["conv1"]] = (0, 2, 1, 2)   # a conv reading blocks writes no bands
    with pytest.raises(ValueError):
        sim.expand(g, bad)
    items, fa, ff, _, an = sim.expand(g, cfg)
    n = len(ts)
    conv1 = next(o["id"] for o in g["ops"] if o["name"] == "conv1")
    assert (2 * n + conv1, 0) in an.temp     # the staged merge of conv1's input
    f_conv1 = next(it for it in items if it.kind == "F" and it.op == conv1)
    assert sorted(f_conv1.reads) == [(nm["pool1"], 0), (nm["pool1"], 1)]
