"""ORACLE — test infrastructure only.

Brute-force plan enumeration on tiny graphs:
  * enumerate every per-tensor configuration opt x p_num of a small DFG
    (Eq. 1's search space restricted to tensors produced by ops);
  * for each, the simulator's peak must equal an independent live-set sum
    recomputed from the item list and the lifetime intervals of the trace, and
    no two live ranges may overlap in the pool;
  * the minimum peak over all plans decides feasibility of a budget (T8: the
    planner may only report INFEASIBLE when no enumerated plan fits).
"""

from __future__ import annotations

import itertools

from . import sim


def act_tensors(graph):
    an = sim.analyze(graph)
    return [t["id"] for t in graph["tensors"] if t["kind"] == "act" and not an.is_loss[t["id"]]]


def enumerate_plans(graph, opts=(0, 1, 2), ps=(1, 2), limit=None):
    acts = act_tensors(graph)
    choices = [(o, p) for o in opts for p in ps
               if p == 1 or graph["samples"] % p == 0]
    count = 0
    for combo in itertools.product(choices, repeat=len(acts)):
        cfg = sim.default_cfg(graph)
        for t, (o, p) in zip(acts, combo):
            cfg[t] = (o, p, 1)
        yield cfg
        count += 1
        if limit and count >= limit:
            return


def independent_peak(res: sim.SimResult):
    """Peak live bytes recomputed from the trace's alloc/free intervals, and a
    check that simultaneously-live ranges never overlap."""
    intervals = []   # (alloc_seq, free_seq, offset, bytes)
    open_ = {}
    for seq, item, kind, key, j, off, b in res.trace:
        if kind == "A":
            open_[(key, j)] = (seq, item, off, b)
        else:
            s0, i0, o0, b0 = open_.pop((key, j))
            assert o0 == off and b0 == b
            intervals.append((i0, item, off, sim.align(b)))
    n_items = len(res.items)
    best = 0
    for i in range(-1, n_items):
        # live during item i: allocated at an item <= i and freed at an item >= i
        live = [(off, b) for (a, f, off, b) in intervals if a <= i <= f and not (f == i and a == i and False)]
        # a piece freed after item f is live during f; allocated at item a is live during a
        tot = sum(b for _, b in live)
        best = max(best, tot)
        live.sort()
        for (o1, b1), (o2, _) in zip(live, live[1:]):
            assert o1 + b1 <= o2, "overlapping live ranges"
    return res.static + best


def min_peak(graph, **kw):
    best = None
    for cfg in enumerate_plans(graph, **kw):
        r = sim.simulate(graph, cfg)
        if best is None or r.peak_extent < best[0]:
            best = (r.peak_extent, cfg)
    return best
