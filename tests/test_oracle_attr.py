"""Attribute (height) splits, reading D-ATTR (Fig. 10, Fig. 6):
the staged-row geometry against a brute-force scan of the direct convolution loop, any band /
sample / swap / recompute plan computing the unsplit gradients (T1) in fp64, and the pool
trace accounting for the staging temporaries."""

import random

import numpy as np
import pytest

from conftest import rel_errs
from oracle import execplan, net, sim
from tsinputs import gen, graphs


def _rows_touched(H, R, s, pad, out_lo, out_hi):
    """Input rows the direct window loop (ops.conv2d_fwd docstring: X[n, p*st + r - pad])
    reads for output rows [out_lo, out_hi), padding rows included."""
    rows = {p * s + r - pad for p in range(out_lo, out_hi) for r in range(R)}
    return min(rows), max(rows)


@pytest.mark.parametrize("H,R,s,pad,P", [(8, 3, 1, 1, 2), (8, 3, 1, 1, 4), (32, 7, 2, 3, 4), (16, 1, 2, 0, 2),
                                        (16, 3, 2, 1, 4), (8, 2, 2, 0, 2), (16, 3, 2, 1, 2), (12, 1, 1, 0, 3)])
def test_band_rows_equal_the_direct_loop(H, R, s, pad, P):
    Ho = (H + 2 * pad - R) // s + 1
    ts = [{"shape": (1, H, H, 4)}, {"shape": (4, R, R, 4)}, {"shape": (1, Ho, Ho, 4)}]
    conv = {"kind": "conv2d", "inputs": [0, 1], "outputs": [2], "iattrs": [s, pad]}
    pool = {"kind": "maxpool", "inputs": [0], "outputs": [2], "iattrs": [R, s, pad]}
    hb = Ho // P
    for op in (conv, pool):
        assert sim.window_geom(op, ts) == (R, s, pad)
        for k in range(P):
            lo, hi, hs = sim.band_rows(op, ts, k, P)
            assert (lo, hi) == _rows_touched(H, R, s, pad, k * hb, (k + 1) * hb)
            assert hs == hi - lo + 1 and (hs - R) // s + 1 == hb   # the unpadded window op yields the band


@pytest.mark.parametrize("H,W,R,S,s,pad,P", [(8, 12, 3, 3, 1, 1, 4), (16, 8, 7, 7, 2, 3, 2), (12, 16, 1, 1, 2, 0, 4)])
def test_width_and_rect_geometry(H, W, R, S, s, pad, P):
    """The staged rectangle of a width band (columns by the direct loop, every row) and of a
    full merge (every row and column the output reads)."""
    Ho, Wo = (H + 2 * pad - R) // s + 1, (W + 2 * pad - S) // s + 1
    g = {"samples": 2, "tensors": [{"shape": (2, H, W, 4), "kind": "act"}, {"shape": (4, R, S, 4), "kind": "param"},
                                   {"shape": (2, Ho, Wo, 4), "kind": "act"}],
         "ops": [{"kind": "conv2d", "inputs": [0, 1], "outputs": [2], "iattrs": [s, pad]}]}
    wb = Wo // P
    cfg = {0: (0, 1, 1), 1: (0, 1, 1), 2: (0, P, 1, 3)}
    for k in range(P):
        rlo, hs, clo, ws, nb = sim.staged_rect(g, cfg, 0, k, P)
        assert (rlo, rlo + hs - 1) == _rows_touched(H, R, s, pad, 0, Ho)
        assert (clo, clo + ws - 1) == _rows_touched(W, S, s, pad, k * wb, (k + 1) * wb)
        assert nb == 2 and (ws - S) // s + 1 == wb and (hs - R) // s + 1 == Ho
    cfg[2] = (0, 2, 1, 0)   # sample split of the output: a full merge of 1 sample per micro-op
    rlo, hs, clo, ws, nb = sim.staged_rect(g, cfg, 0, 1, 2)
    assert (rlo, hs, clo, ws, nb) == (-pad, (Ho - 1) * s + R, -pad, (Wo - 1) * s + S, 1)


def _components(g):
    """Groups of 4-D activations joined by band-local ops (they must share one band split)."""
    ts, ops = g["tensors"], g["ops"]
    parent = {t["id"]: t["id"] for t in ts if t["kind"] == "act" and len(t["shape"]) == 4}

    def find(a):
        while parent[a] != a:
            a = parent[a]
        return a
    for o in ops:
        if o["kind"] in sim.ATTR_LOCAL:
            for x in o["inputs"]:
                if x in parent:
                    parent[find(x)] = find(o["outputs"][0])
    comp = {}
    for t in parent:
        comp.setdefault(find(t), []).append(t)
    return list(comp.values())


def _draw_attr_cfg(g, r, ps, dims):
    """A random legal plan with band splits: memory options at random, then each group of
    band-joined tensors in turn takes a height or width band split, a sample split or none
    when legal."""
    ts = g["tensors"]
    acts = [t["id"] for t in ts if t["kind"] == "act" and t["name"] != "loss"]
    cfg = {t["id"]: (0, 1, 1) for t in ts}
    for t in acts:
        cfg[t] = (r.choice([0, 1, 2]), 1, 1)
    comps = _components(g)
    r.shuffle(comps)
    for comp in comps:
        mode = r.choice(["band", "band", "sample", "none"])
        p, d = r.choice(ps), r.choice(dims)
        trial = dict(cfg)
        for t in comp:
            opt = cfg[t][0]
            trial[t] = (opt, p, 1, d) if mode == "band" else (opt, p, 1, 0) if mode == "sample" else (opt, 1, 1)
        try:
            sim.expand(g, trial)
            cfg = trial
        except ValueError:
            pass
    for t in acts:   # the rest of the 2-D tensors: sample splits
        if len(ts[t]["shape"]) != 4 and cfg[t][1] == 1 and r.random() < 0.5:
            trial = dict(cfg)
            trial[t] = (cfg[t][0], 2, 1)
            try:
                sim.expand(g, trial)
                cfg = trial
            except ValueError:
                pass
    return cfg


def _rand_attr_cfg(g, r, ps=(2, 4), dims=(2, 3)):
    for _ in range(20):
        cfg = _draw_attr_cfg(g, r, ps, dims)
        if any(sim.is_attr(g, cfg, t) for t in cfg):
            return cfg
    raise AssertionError("no band split drawn")


@pytest.mark.parametrize("gname,seed", [("vgg_tiny", 0), ("vgg_tiny", 1), ("resnet_tiny", 0), ("resnet_tiny", 1),
                                        ("resnet_tiny", 2)])
def test_t1_band_plans_compute_the_unsplit_gradients(gname, seed):
    g = graphs.config_graph(gname, dtype="f32")
    P, I = gen.init_params(g), gen.make_inputs(g)
    loss, pg, _, _ = net.train_step(g, P, I)
    r = random.Random(seed)
    for trial in range(2):
        cfg = _rand_attr_cfg(g, r)
        l2, pg2 = execplan.execute(g, cfg, P, I, cache_bytes=r.choice([0, 1 << 20]))
        assert abs(l2 - loss) <= 1e-12 * abs(loss)
        assert max(rel_errs(pg2, pg).values()) <= 1e-12


def test_batch1_band_split_lowers_the_peak():
    """Fig. 6: at batch 1 the sample dim cannot be split; splitting the height
    lowers the swapped plan's peak, staging temporaries included."""
    g = graphs.config_graph("vgg_tiny", dtype="f32", batch=1)
    comps = _components(g)
    base = {t["id"]: (0, 1, 1) for t in g["tensors"]}
    acts = [t["id"] for t in g["tensors"] if t["kind"] == "act" and t["name"] != "loss"]
    for t in acts:
        base[t] = (sim.SWAP, 1, 1)
    band = dict(base)
    for comp in comps:
        trial = dict(band)
        for t in comp:
            trial[t] = (sim.SWAP, 4, 1, 2)
        try:
            sim.expand(g, trial)
            band = trial
        except ValueError:   # the group feeding the flatten stays whole
            pass
    r0 = sim.simulate(g, base)
    r1 = sim.simulate(g, band)
    assert r1.peak_live < r0.peak_live
    temps = [e for e in r1.trace if e[3] >= 2 * len(g["tensors"])]
    assert temps and all(e[6] > 0 for e in temps)
    # every temporary is freed by the item that allocated it
    seen = {}
    for seq, item, kind, key, j, off, nb in temps:
        if kind == "A":
            seen[(key, j)] = item
        else:
            assert seen.pop((key, j)) == item
    assert not seen


def test_band_split_legality():
    g = graphs.config_graph("vgg_tiny", dtype="f32")
    ts = g["tensors"]
    byname = {t["name"]: t["id"] for t in ts}
    cfg = {t["id"]: (0, 1, 1) for t in ts}
    cfg[byname["conv0"]] = (0, 2, 1, 2)   # relu0 reads it: a band-local consumer needs the same split
    with pytest.raises(ValueError):
        sim.expand(g, cfg)
    cfg[byname["relu0"]] = (0, 2, 1, 2)
    sim.expand(g, cfg)
    cfg[byname["relu0"]] = (0, 4, 1, 2)
    with pytest.raises(ValueError):
        sim.expand(g, cfg)
    last = [t for t in ts if t["kind"] == "act" and len(t["shape"]) == 4][-1]   # read by flatten
    cfg2 = {t["id"]: (0, 1, 1) for t in ts}
    cfg2[last["id"]] = (0, 2, 1, 2)
    with pytest.raises(ValueError):
        sim.expand(g, cfg2)
    cfg3 = {t["id"]: (0, 1, 1) for t in ts}
    cfg3[byname["conv0"]] = (0, 3, 1, 2)  # H % p != 0
    cfg3[byname["relu0"]] = (0, 3, 1, 2)
    with pytest.raises(ValueError):
        sim.expand(g, cfg3)


def stride2_graph(dtype="f32"):
    """X [2, 8, 8, 8] -> conv a 3x3 / 1 -> relu -> conv b 1x1 / 2 -> flatten -> fc -> loss: with
    relu's output in 8 one-row bands, conv b (unsplit output: a full merge) stages rows 0 .. 6
    (and reads only the even ones), so band 7 is staged by no micro-op: its gradient is zero
    without any writer."""
    b = graphs.GraphBuilder("vgg_stride2", dtype, 2)  # (CNN parameter recipe)
    X = b.tensor("X", (2, 8, 8, 8), "input")
    Y = b.tensor("labels", (2,), "label", dtype="i32")
    Wa, ba = b.param("Wa", (8, 3, 3, 8)), b.param("ba", (8,))
    Wb, bb = b.param("Wb", (8, 1, 1, 8)), b.param("bb", (8,))
    Wf, bf = b.param("Wf", (3, 128)), b.param("bf", (3,))
    a = b.op("conv2d", "conv_a", [X, Wa, ba], (2, 8, 8, 8), iattrs=[1, 1])
    r = b.op("relu", "relu", [a], (2, 8, 8, 8))
    c = b.op("conv2d", "conv_b", [r, Wb, bb], (2, 4, 4, 8), iattrs=[2, 0])
    f = b.op("flatten", "flat", [c], (2, 128))
    y = b.op("linear", "fc", [f, Wf, bf], (2, 3))
    b.op("xent", "loss", [y, Y], (1,), out_dtype="f32")
    g = b.done()
    cfg = sim.default_cfg(g)
    cfg[a] = (sim.RESIDE, 8, 1, 2)
    cfg[r] = (sim.RESIDE, 8, 1, 2)
    return g, cfg


def test_bands_no_window_reaches_have_zero_gradient():
    g, cfg = stride2_graph()
    items, fa, ff, _, an = sim.expand(g, cfg)
    n = len(g["tensors"])
    conv_b = next(o["id"] for o in g["ops"] if o["name"] == "conv_b")
    relu = next(t["id"] for t in g["tensors"] if t["name"] == "relu")
    written = {j for it in items if it.kind == "B" and it.op == conv_b for (key, j) in it.writes if key == n + relu}
    assert written == set(range(7))   # the staged rectangle spans rows 0..6: band 7 is unread
    reads = {j for it in items if it.kind == "F" and it.op == conv_b for (key, j) in it.reads if key == relu}
    assert reads == set(range(7))
    # drelu.7 is first touched by relu's backward reading it: allocated as zeros
    b_relu = [it for it in items if it.kind == "B" and g["ops"][it.op]["name"] == "relu"]
    assert {j for it in b_relu for (key, j) in it.reads if key == n + relu} == set(range(8))
    P, I = gen.init_params(g), gen.make_inputs(g)
    loss, pg, _, _ = net.train_step(g, P, I)
    l2, pg2 = execplan.execute(g, cfg, P, I)
    assert abs(l2 - loss) <= 1e-12 * abs(loss)
    assert max(rel_errs(pg2, pg).values()) <= 1e-12
