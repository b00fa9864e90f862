"""Data-parallel host path on CPU (world_size 2, gloo): rank 0 plans and broadcasts
the serialized plan, every rank rebuilds the identical augmented schedule and
allocation trace (all ranks execute the same plan, so NCCL calls
are issued in the same order), and the max-over-ranks timing reduction."""

import os

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _worker(rank, world, port, q, gname="bert_tiny"):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icde_niemyc22_b200 import tsplit
        from tsinputs import graphs
        if gname == "mlp_b1":  # batch 1: the planner splits channels (reading D-CH)
            g = graphs.mlp(batch=1, in_dim=64, hidden=2048, depth=3, classes=10)
            base = tsplit.Plan.default(tsplit.Graph(g)).stats()
            budget = base["static_bytes"] + (base["peak_extent"] - base["static_bytes"]) * 3 // 4
        else:
            g = graphs.config_graph("bert_tiny")
            base = tsplit.Plan.default(tsplit.Graph(g)).stats()
            budget = base["static_bytes"] + (base["peak_extent"] - base["static_bytes"]) // 3
        G = tsplit.Graph(g)
        blob = tsplit.Plan.plan(G, budget).serialize() if rank == 0 else None
        obj = [blob]
        dist.broadcast_object_list(obj, src=0)
        plan = tsplit.Plan.deserialize(G, obj[0])
        trace = plan.trace()
        items = plan.items()
        # every rank holds the same schedule: compare a digest across ranks
        import hashlib
        buckets = plan.grad_buckets(1 << 14)  # NCCL call order must match across ranks
        h = hashlib.sha1(repr((trace, items, buckets)).encode()).hexdigest()
        digest = torch.tensor([int(h[:15], 16)], dtype=torch.int64)
        gathered = [torch.zeros_like(digest) for _ in range(world)]
        dist.all_gather(gathered, digest)
        # max-over-ranks step time (bench.py reduction)
        t = torch.tensor([0.1 * (rank + 1)], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        dims = sorted({plan.get_dim(t["id"]) for t in g["tensors"] if t["kind"] == "act"})
        q.put((rank, [int(x.item()) for x in gathered], float(t.item()), plan.stats()["peak_extent"] <= budget, dims))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("gname", ["bert_tiny", "mlp_b1"])
def test_plan_broadcast_world2(gname):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + (os.getpid() % 1000) + (7 if gname == "mlp_b1" else 0)
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, gname)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in procs]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, digests, tmax, fits, dims in res:
        assert len(set(digests)) == 1, digests
        assert tmax == pytest.approx(0.2)
        assert fits
        if gname == "mlp_b1":
            assert 1 in dims  # the broadcast plan carries the channel dim
