"""Data-parallel gradient buckets, host logic on CPU:
the spans of all buckets tile the gradient region exactly once, every parameter's
bucket is launched no earlier than the last backward micro-op that writes its
gradient (dW merges across splits by summation), buckets are emitted in
schedule order, and a smaller bucket size gives more, earlier buckets."""

import pytest

from paper_conf_icde_niemyc22_b200 import tsplit
from tsinputs import graphs


def _param_layout(g):
    """(offset, aligned bytes) of every parameter gradient: fp32, 256-B aligned,
    in tensor-id order after masters (+ bf16 copies) — DESIGN.md §5."""
    ps = [t for t in g["tensors"] if t["kind"] == "param"]
    al = lambda b: (b + 255) // 256 * 256  # noqa: E731
    n = lambda t: int(__import__("numpy").prod(t["shape"]))  # noqa: E731
    off = sum(al(4 * n(t)) for t in ps)
    if g["dtype"] == "bf16":
        off += sum(al(2 * n(t)) for t in ps)
    out = {}
    for t in ps:
        out[t["id"]] = (off, al(4 * n(t)))
        off += al(4 * n(t))
    return out


@pytest.mark.parametrize("name,frac", [("bert_tiny", 0.4), ("resnet_tiny", 0.7), ("mlp", None)])
@pytest.mark.parametrize("bucket", [1 << 10, 1 << 16, 1 << 30])
def test_buckets_tile_grads_after_last_writer(name, frac, bucket):
    g = graphs.config_graph(name)
    G = tsplit.Graph(g)
    P = tsplit.Plan.default(G)
    if frac is not None:
        st = P.stats()
        P = tsplit.Plan.plan(G, st["static_bytes"] + int(frac * (st["peak_extent"] - st["static_bytes"])))
    spans = P.grad_buckets(bucket)
    layout = _param_layout(g)
    # exact tiling of the gradient region
    lo = min(o for o, _ in layout.values())
    hi = max(o + b for o, b in layout.values())
    cov = sorted((o, b) for _, o, b in spans)
    pos = lo
    for o, b in cov:
        assert o == pos, (o, pos)
        pos += b
    assert pos == hi
    # launch point >= last writer of every parameter inside the span
    items = P.items()
    last = {}
    for i, (kind, op, k, aux) in enumerate(items):
        if kind == "B":
            for x in g["ops"][op]["inputs"]:
                if g["tensors"][x]["kind"] == "param":
                    last[x] = i
    for after, o, b in spans:
        for tid, (po, pb) in layout.items():
            if o <= po < o + b:
                assert after >= last.get(tid, -1), (tid, after, last.get(tid))
    afters = [a for a, _, _ in spans]
    assert afters == sorted(afters)
    if bucket == 1 << 30:
        assert len(set(afters)) == 1 and afters[0] == len(items) - 1


def test_smaller_buckets_start_earlier():
    g = graphs.config_graph("bert_tiny")
    P = tsplit.Plan.default(tsplit.Graph(g))
    small = P.grad_buckets(1 << 12)
    big = P.grad_buckets(1 << 30)
    assert len({a for a, _, _ in small}) > 1
    assert min(a for a, _, _ in small) < min(a for a, _, _ in big)
