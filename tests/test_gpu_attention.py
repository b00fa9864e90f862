"""Fused attention on the GPU, through the C ABI:

* the tensor-core (mma.sync) and CUDA-core kernels against the fp64 oracle
  (oracle.ops.attention_fwd / attention_bwd) on bf16-representable inputs, with and
  without dropout, several sequence lengths, a nonzero first-sample offset (dropout
  counters of a later micro-op) and accumulate flags;
* a sample split of the kernels equals the whole batch bit for bit;
* whole training steps of the fused tiny BERT: fp32 random plans vs the oracle (1e-5)
  and split vs unsplit (1e-6), bf16 per tensor vs the plain oracle (2e-2), fused vs
  unfused graph.
"""

import random

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from conftest import assert_bf16_parity, global_rel_err, rel_errs  # noqa: E402
from oracle import brute, net, sim  # noqa: E402
from oracle import ops as O  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def _rel(a, b):
    a, b = np.asarray(a, np.float64), np.asarray(b, np.float64)
    return float(np.linalg.norm(a - b) / max(np.linalg.norm(b), 1e-30))


def _inputs(nb, heads, seq, d, seed=0):
    r = np.random.default_rng(seed)
    h = heads * d
    mk = lambda s: gen.snap_bf16((s * r.standard_normal((nb * seq, h))).astype(np.float32))  # noqa: E731
    return mk(1.0), mk(1.0), mk(1.0), mk(1.0)


@pytest.mark.parametrize("seq", [64, 128, 192, 384, 512])
@pytest.mark.parametrize("p", [0.0, 0.1])
@pytest.mark.parametrize("path", ["tc", "mma", "simt"])
def test_attention_kernels_vs_oracle(seq, p, path):
    """path tc: the default dispatch (tcgen05 forward where seq % 128 == 0, else mma.sync);
    mma: the mma.sync forward forced; simt: CUDA cores."""
    nb, heads, d = 2, 3, 64
    alpha, seed, b0, step = 0.125, 77, 5, 3
    q, k, v, dc = _inputs(nb, heads, seq, d)
    c_ref, lse_ref, mask_ref = O.attention_fwd(q, k, v, heads, seq, alpha, p, seed, b0 * heads * seq * seq, step)
    dq_ref, dk_ref, dv_ref = O.attention_bwd(dc, q, k, v, heads, seq, alpha, p, seed, b0 * heads * seq * seq, step)
    dev = lambda a: torch.from_numpy(a).to("cuda").to(torch.bfloat16)  # noqa: E731
    Q, K, V, DC = dev(q), dev(k), dev(v), dev(dc)
    C = torch.empty_like(Q)
    L = torch.empty((nb, heads, seq), dtype=torch.float32, device="cuda")
    M = torch.empty((nb, heads, seq, seq // 32), dtype=torch.int32, device="cuda")
    geom = (nb, heads, seq, d, seed, b0, step)
    force = 0x10 if path == "simt" else 0
    used = tsplit.attention(1 | force, geom, alpha, p, Q, K, V, c=C, lse=L, mask=M, acc=0x100 if path == "mma" else 0)
    torch.cuda.synchronize()
    assert used == {"simt": 0, "mma": 1, "tc": 2 if seq % 128 == 0 else 1}[path]
    assert np.array_equal(M.cpu().numpy(), mask_ref)  # keep bits: integer decisions, bit-exact
    assert _rel(L.cpu().numpy(), lse_ref) <= 1e-5
    assert _rel(C.float().cpu().numpy(), c_ref) <= 1e-2
    ws = torch.empty(nb * heads * seq, dtype=torch.float32, device="cuda")
    dQ, dK, dV = (torch.full_like(Q, 0.25) for _ in range(3))
    mma = 0x100 if path == "mma" else 0
    tsplit.attention(2 | force, geom, alpha, p, Q, K, V, c=C, lse=L, mask=M, dc=DC, dq=dQ, dk=dK, dv=dV, ws=ws,
                     acc=mma)
    torch.cuda.synchronize()
    for got, ref in ((dQ, dq_ref), (dK, dk_ref), (dV, dv_ref)):
        assert _rel(got.float().cpu().numpy(), ref) <= 2e-2
    # accumulate flags (a later backward op adding its share)
    tsplit.attention(2 | force, geom, alpha, p, Q, K, V, c=C, lse=L, mask=M, dc=DC, dq=dQ, dk=dK, dv=dV,
                     acc=7 | mma, ws=ws)
    torch.cuda.synchronize()
    for got, ref in ((dQ, dq_ref), (dK, dk_ref), (dV, dv_ref)):
        assert _rel(got.float().cpu().numpy(), 2 * ref) <= 2e-2


@pytest.mark.parametrize("nb,heads,seq,ramp", [(8, 16, 512, 3.0), (3, 5, 384, 6.0), (2, 2, 1024, 4.0)])
def test_tc_forward_online_rescale_persistent(nb, heads, seq, ramp):
    """The tcgen05 forward streams K/V in 128-key chunks with an online softmax whose running
    max moves only when it grows by > 8 (log2 units).  Keys scaled by a ramp along the sequence
    make later chunks' maxima jump past that threshold (O-row rescale path); (8, 16, 512) has
    256 work items, more than the persistent grid, so CTAs loop over items; seq 384 has an odd
    tile count (single-tile items); seq 1024 exceeds the old whole-row-in-TMEM limit."""
    d, alpha, p, seed, b0, step = 64, 0.5, 0.1, 11, 2, 4
    q, k, v, dc = _inputs(nb, heads, seq, d, seed=5)
    pos = np.tile(np.arange(seq), nb)[:, None]
    k = gen.snap_bf16((k * (1.0 + ramp * pos / seq)).astype(np.float32))
    c_ref, lse_ref, mask_ref = O.attention_fwd(q, k, v, heads, seq, alpha, p, seed, b0 * heads * seq * seq, step)
    # the ramp really crosses the rescale threshold somewhere: chunk maxima grow by > 8 / log2(e)
    s = np.einsum("qhd,khd->hqk", q.reshape(nb * seq, heads, d)[:seq], k.reshape(nb * seq, heads, d)[:seq]) * alpha
    cm = s.reshape(heads, seq, seq // 128, 128).max(-1)
    assert (np.diff(np.maximum.accumulate(cm, axis=-1), axis=-1) > 8 / np.log2(np.e)).any()
    dev = lambda a: torch.from_numpy(a).to("cuda").to(torch.bfloat16)  # noqa: E731
    Q, K, V = dev(q), dev(k), dev(v)
    C = torch.empty_like(Q)
    L = torch.empty((nb, heads, seq), dtype=torch.float32, device="cuda")
    M = torch.empty((nb, heads, seq, seq // 32), dtype=torch.int32, device="cuda")
    used = tsplit.attention(1, (nb, heads, seq, d, seed, b0, step), alpha, p, Q, K, V, c=C, lse=L, mask=M)
    torch.cuda.synchronize()
    assert used == 2
    assert np.array_equal(M.cpu().numpy(), mask_ref)
    assert _rel(L.cpu().numpy(), lse_ref) <= 1e-5
    assert _rel(C.float().cpu().numpy(), c_ref) <= 1e-2


def test_attention_split_equals_whole():
    """Two micro-ops of 2 samples each (b0 = 0, 2) reproduce the 4-sample call bit for bit."""
    nb, heads, seq, d = 4, 2, 128, 64
    q, k, v, dc = _inputs(nb, heads, seq, d, seed=4)
    dev = lambda a: torch.from_numpy(a).to("cuda").to(torch.bfloat16)  # noqa: E731
    Q, K, V, DC = dev(q), dev(k), dev(v), dev(dc)
    C, C2 = torch.empty_like(Q), torch.empty_like(Q)
    L, L2 = (torch.empty((nb, heads, seq), dtype=torch.float32, device="cuda") for _ in range(2))
    M, M2 = (torch.empty((nb, heads, seq, seq // 32), dtype=torch.int32, device="cuda") for _ in range(2))
    ws = torch.empty(nb * heads * seq, dtype=torch.float32, device="cuda")
    G = [torch.empty_like(Q) for _ in range(6)]
    tsplit.attention(1, (nb, heads, seq, d, 9, 0, 1), 0.125, 0.1, Q, K, V, c=C, lse=L, mask=M)
    tsplit.attention(2, (nb, heads, seq, d, 9, 0, 1), 0.125, 0.1, Q, K, V, c=C, lse=L, mask=M, dc=DC, dq=G[0],
                     dk=G[1], dv=G[2], ws=ws)
    rows = seq * 2
    for s0 in (0, 2):
        sl = slice(s0 * seq, s0 * seq + rows)
        g2 = (2, heads, seq, d, 9, s0, 1)
        tsplit.attention(1, g2, 0.125, 0.1, Q[sl], K[sl], V[sl], c=C2[sl], lse=L2[s0:s0 + 2], mask=M2[s0:s0 + 2])
        tsplit.attention(2, g2, 0.125, 0.1, Q[sl], K[sl], V[sl], c=C2[sl], lse=L2[s0:s0 + 2], mask=M2[s0:s0 + 2],
                         dc=DC[sl], dq=G[3][sl], dk=G[4][sl], dv=G[5][sl], ws=ws)
    torch.cuda.synchronize()
    assert torch.equal(C, C2) and torch.equal(L, L2) and torch.equal(M, M2)
    for i in range(3):
        assert torch.equal(G[i], G[3 + i])


def _run(g, plan_cfg=None, budget=None):
    G = tsplit.Graph(g)
    if budget is not None:
        P = tsplit.Plan.plan(G, budget)
    else:
        P = tsplit.Plan.default(G)
        for t, (o, p, lead) in (plan_cfg or {}).items():
            P.set(t, o, p, lead)
    S = tsplit.Session(G, P)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    S.set_params(params)
    loss = S.step(tsplit.inputs_to_device(G, inputs))
    return loss, S.grads(), S, P


@pytest.mark.parametrize("seed", range(3))
def test_fused_bert_tiny_fp32_random_plans(seed):
    g = graphs.config_graph("bert_tiny", dtype="f32", fused_attention=True)
    r = random.Random(seed)
    cfg = {t: (r.choice([0, 1, 2]), r.choice([1, 2, 4]), r.choice([1, 2])) for t in brute.act_tensors(g)}
    loss, grads, S, P = _run(g, cfg)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    ol, og, _, _ = net.train_step(g, params, inputs)
    assert abs(loss - ol) <= 1e-5 * abs(ol)
    errs = rel_errs(grads, og)
    assert max(errs.values()) <= 1e-5, sorted(errs.items(), key=lambda kv: -kv[1])[:5]
    l0, g0, _, _ = _run(g)
    assert max(rel_errs(grads, g0).values()) <= 1e-6
    assert S.trace() == [tuple(e) for e in sim.simulate(g, {**sim.default_cfg(g), **cfg}).trace]


@pytest.mark.parametrize("seq", [128, 192])
def test_fused_bert_small_bf16_tensor_cores(seq):
    """Head dim 64: seq 128 runs the tcgen05 kernels inside the session, seq 192 (not a
    multiple of 128) the mma.sync ones.  Per tensor within 2e-2 of the plain fp64 oracle
    (R17); fused = unfused graph within the same bar; a budgeted plan trains the same
    function."""
    g = graphs.config_graph("bert_small", seq=seq, fused_attention=True)
    gu = graphs.config_graph("bert_small", seq=seq)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    ol, og, _, _ = net.train_step(g, params, inputs)
    loss, grads, S, P = _run(g)
    assert abs(loss - ol) <= 2e-2 * abs(ol)
    assert_bf16_parity(grads, og)
    lu, gu_, _, _ = _run(gu)
    assert_bf16_parity(gu_, og)
    base = P.stats()
    budget = base["static_bytes"] + (base["peak_extent"] - base["static_bytes"]) * 4 // 10
    l2, g2, S2, P2 = _run(g, budget=budget)
    assert P2.stats()["peak_extent"] <= budget
    assert S2.trace() == P2.trace()
    assert_bf16_parity(g2, og)
    import os
    os.environ["TSPLIT_NO_FUSION"] = "1"  # plan invariance with both programs unfused (D-QKV)
    try:
        _, u0, _, _ = _run(g)
        _, u2, _, _ = _run(g, budget=budget)
    finally:
        os.environ.pop("TSPLIT_NO_FUSION", None)
    assert global_rel_err(u2, u0) <= 1e-6


def test_tc_forward_partial_outputs_for_replays():
    """A recompute replay regenerates only the output it targets (C, or lse, or the keep
    bits): the tcgen05 forward runs with the other pointers null (it used to fall back to
    the mma.sync kernel) and writes exactly what the full call writes."""
    nb, heads, seq, d = 2, 3, 256, 64
    q, k, v, _ = _inputs(nb, heads, seq, d, seed=8)
    dev = lambda a: torch.from_numpy(a).to("cuda").to(torch.bfloat16)  # noqa: E731
    Q, K, V = dev(q), dev(k), dev(v)
    geom = (nb, heads, seq, d, 21, 1, 2)
    C = torch.empty_like(Q)
    L = torch.empty((nb, heads, seq), dtype=torch.float32, device="cuda")
    M = torch.empty((nb, heads, seq, seq // 32), dtype=torch.int32, device="cuda")
    assert tsplit.attention(1, geom, 0.125, 0.1, Q, K, V, c=C, lse=L, mask=M) == 2
    C2, L2, M2 = torch.zeros_like(C), torch.zeros_like(L), torch.zeros_like(M)
    assert tsplit.attention(1, geom, 0.125, 0.1, Q, K, V, c=C2) == 2
    assert tsplit.attention(1, geom, 0.125, 0.1, Q, K, V, lse=L2) == 2
    assert tsplit.attention(1, geom, 0.125, 0.1, Q, K, V, mask=M2) == 2
    torch.cuda.synchronize()
    assert torch.equal(C, C2) and torch.equal(L, L2) and torch.equal(M, M2)


def test_attention_backward_in_workspace_chunks():
    """A fused-attention micro-op whose row terms D = rowsum(dO * O) exceed the workspace
    (h1024 a16 s512: 255 samples fit; an unsplit batch of 288) runs its backward in sample
    chunks; the step equals the plan whose micro-ops hold 144 samples (no chunking)."""
    g = graphs.bert(layers=1, hidden=1024, heads=16, seq=512, batch=288, vocab=512, fused_attention=True)
    l0, g0, S0, _ = _run(g)
    cfg = {t: (0, 2, 1) for t in brute.act_tensors(g)}
    l1, g1, S1, _ = _run(g, cfg)
    assert abs(l0 - l1) <= 1e-3 * abs(l1)
    assert global_rel_err(g0, g1) <= 1e-3
