"""Data parallelism on one GPU (north_star: DP over NVLink, each GPU on
its own split plan and PCIe link).  The round's box has one GPU, so the N ranks run as N
sessions in one process: rank 0 plans and serializes, every rank deserializes the same
plan, each rank steps on its own shard with its global sample offset, and the gradients
are summed and scaled by 1/world — exactly what the per-bucket ncclAllReduce plus the
SGD's 1/world scale compute (the NCCL path itself: test_gpu_session's 1-rank test).
The result must be the oracle's step over the concatenated batch (R14, R15)."""

import random

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from conftest import assert_bf16_parity, global_rel_err, rel_errs  # noqa: E402
from oracle import brute, net  # noqa: E402
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402
from tsinputs import gen, graphs  # noqa: E402


def _shard_oracle(name, dtype, fused, params, inputs, sample0):
    """fp64 step of one shard whose samples sit at global index sample0 (the dropout
    counters, R15, follow global sample indices).  The oracle has no offset argument, and
    BERT couples no samples (per-row / per-sample ops), so: step [pad; shard] and pad alone
    and difference the gradient sums — the shard's own mean gradient, at its offset."""
    b = graphs.config_graph(name, dtype=dtype, fused_attention=fused)["samples"]
    if sample0 == 0:
        return net.train_step(graphs.config_graph(name, dtype=dtype, fused_attention=fused), params, inputs)[1]
    gp = graphs.config_graph(name, dtype=dtype, fused_attention=fused, batch=sample0)
    big = graphs.config_graph(name, dtype=dtype, fused_attention=fused, batch=sample0 + b)
    pad = gen.make_inputs(gp, seed=99)
    _, og_big, _, _ = net.train_step(big, params, _concat(big, [pad, inputs]))
    _, og_pad, _, _ = net.train_step(gp, params, pad)
    return {k: ((sample0 + b) * og_big[k] - sample0 * og_pad[k]) / b for k in og_big}


def _concat(graph_global, shards):
    out = {}
    for t in graph_global["tensors"]:
        if t["kind"] in ("input", "label"):
            out[t["name"]] = np.concatenate([s[t["name"]] for s in shards], axis=0)
    return out


@pytest.mark.parametrize("dtype,fused", [("f32", True), ("f32", False), ("bf16", True)])
@pytest.mark.parametrize("world", [2, 4])
def test_shards_sum_to_the_concatenated_batch(dtype, fused, world):
    name = "bert_tiny" if dtype == "f32" else "bert_small"
    g = graphs.config_graph(name, dtype=dtype, fused_attention=fused)          # per-rank batch b
    b = g["samples"]
    gg = graphs.config_graph(name, dtype=dtype, fused_attention=fused, batch=b * world)  # global
    params = gen.init_params(g)
    shards = [gen.make_inputs(g, seed=r) for r in range(world)]  # rank seeds (SURVEY C4 inputs)
    G = tsplit.Graph(g)
    r = random.Random(world)
    cfg = {t: (r.choice([0, 1, 2]), r.choice([1, 2]), 1) for t in brute.act_tensors(g)}
    P0 = tsplit.Plan.default(G)
    for t, c in cfg.items():
        P0.set(t, *c)
    blob = P0.serialize()  # rank 0 -> broadcast -> every rank
    total, losses = None, []
    for rank in range(world):
        P = tsplit.Plan.deserialize(G, blob)
        S = tsplit.Session(G, P, world_size=world, sample_offset=rank * b)
        S.set_params(params)
        losses.append(S.step(tsplit.inputs_to_device(G, shards[rank])))
        gr = S.grads()
        total = gr if total is None else {k: total[k] + gr[k] for k in gr}
        del S
        if dtype == "bf16":  # each rank within the bf16 bar of its own shard's fp64 step
            assert_bf16_parity(gr, _shard_oracle(name, dtype, fused, params, shards[rank], rank * b))
    dp = {k: v / world for k, v in total.items()}
    ol, og, _, _ = net.train_step(gg, params, _concat(gg, shards))
    assert abs(sum(losses) / world - ol) <= (1e-5 if dtype == "f32" else 2e-2) * abs(ol)
    if dtype == "f32":  # the composition is exact: sum x 1/world = the concatenated batch
        errs = rel_errs(dp, og)
        assert max(errs.values()) <= 1e-5, sorted(errs.items(), key=lambda kv: -kv[1])[:3]
    else:  # bf16: each rank held to the bar above; the mean carries their rounding (D-TOL)
        assert global_rel_err(dp, og) <= 2e-2


def test_ranks_draw_disjoint_dropout_masks():
    """With the global sample offset, rank 1's masks are those of samples b..2b-1 of the
    global batch — not a copy of rank 0's (the same shard stepped at offsets 0 and b gives
    different gradients; at equal offsets, identical ones)."""
    g = graphs.config_graph("bert_tiny", dtype="f32", fused_attention=True)
    G = tsplit.Graph(g)
    P = tsplit.Plan.default(G)
    params, inputs = gen.init_params(g), gen.make_inputs(g)
    dev = tsplit.inputs_to_device(G, inputs)
    out = []
    for off in (0, 0, g["samples"]):
        S = tsplit.Session(G, P, sample_offset=off)
        S.set_params(params)
        S.step(dev)
        out.append(S.grads())
        del S
    # equal offsets: identical except the word-table gradient, whose fp32 atomicAdd order varies
    # from run to run (measured up to 8e-9 relative)
    assert max(rel_errs(out[1], out[0]).values()) <= 1e-7
    assert max(rel_errs(out[2], out[0]).values()) > 1e-3


def test_swap_pool_is_numa_local():
    """The pinned swap pool holds exactly the plan's swapped pieces and, where sysfs names
    the GPU's NUMA node, its pages are bound there (per-rank host memory is reported)."""
    g = graphs.config_graph("bert_small", fused_attention=True)
    names = {t["name"]: t["id"] for t in g["tensors"]}
    G = tsplit.Graph(g)
    P = tsplit.Plan.default(G)
    P.set(names["l0.ffn1"], tsplit.SWAP, 2, 1)
    P.set(names["l1.ctx"], tsplit.SWAP, 1, 1)
    S = tsplit.Session(G, P)
    nbytes, node = S.host_pool()
    assert nbytes >= P.stats()["d2h_bytes"] > 0
    bus = torch.cuda.get_device_properties(0)
    try:
        pci = "%04x:%02x:%02x.0" % (bus.pci_domain_id, bus.pci_bus_id, bus.pci_device_id)
        want = int(open(f"/sys/bus/pci/devices/{pci}/numa_node").read())
    except (OSError, AttributeError, ValueError):
        want = -1
    print("swap pool", nbytes, "B on NUMA node", node, "(GPU's node per sysfs:", want, ")")
    if want >= 0:
        assert node == want
    S.set_params(gen.init_params(g))
    S.step(tsplit.inputs_to_device(G, gen.make_inputs(g)))
    assert S.trace() == P.trace()
