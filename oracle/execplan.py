"""ORACLE — test infrastructure only.

Executes an augmented schedule (sim.expand) piece by piece in fp64: every
micro-op runs the plain op definition (oracle.ops via oracle.net) on its block
of samples, swap-out moves a piece to a host dict, swap-in moves it back, a
recompute replay re-runs the producer micro-op, and a freed piece is deleted.
A read of a piece that is not resident raises.  Pins SURVEY.md §4 T1 / P:L42:
any split/swap/recompute plan yields the gradients of unsplit execution.
"""

from __future__ import annotations

import numpy as np

from . import net, sim
from . import ops as O

F = np.float64


def execute(graph, cfg, params, inputs, step=0, cache_bytes=0):
    items, f_alloc, f_free, fwd_end, an = sim.expand(graph, cfg, cache_bytes=cache_bytes)
    ts, ops = graph["tensors"], graph["ops"]
    n, B = an.n, graph["samples"]
    pval = {t["id"]: np.asarray(params[t["name"]], F) for t in ts if t["kind"] == "param"}
    pgrad = {tid: np.zeros_like(v) for tid, v in pval.items()}
    store, host = {}, {}

    def p_of(t):
        return cfg[t][1] if (an.sample[t] and ts[t]["kind"] == "act") else 1

    def chan(t):  # channel-split (D-CH): p blocks of columns, each over every sample
        return an.sample[t] and ts[t]["kind"] == "act" and sim.dim_of(cfg, t) == 1 and p_of(t) > 1

    def cmode(o):
        return any(chan(t) for t in ops[o]["outputs"])

    def rows_per_sample(t):
        return ts[t]["shape"][0] // B

    def band(t):  # attribute split (D-ATTR): p bands of rows (columns), each over every sample
        return an.sample[t] and sim.is_attr(graph, cfg, t)

    def amode(o):
        return any(band(t) for t in ops[o]["outputs"])

    def staged(o):
        x = ops[o]["inputs"][0]
        return ops[o]["kind"] in sim.ATTR_WINDOW and (band(x) or amode(o) or (ops[o]["kind"] == "conv2d" and chan(x)))

    def piece_shape(t):
        sh = list(ts[t]["shape"])
        if chan(t):
            sh[-1] //= p_of(t)
        elif band(t):
            sh[sim.axis_of(cfg, t)] //= p_of(t)
        elif an.sample[t]:
            sh[0] //= p_of(t)
        return tuple(sh)

    for t in ts:
        if t["kind"] in ("input", "label"):
            a = np.asarray(inputs[t["name"]])
            store[(t["id"], 0)] = a.astype(np.int64) if t["dtype"] == "i32" else a.astype(F)

    def P_op(o):
        if cmode(o):
            return max(p_of(t) for t in ops[o]["outputs"] if chan(t))
        if amode(o):
            return max(p_of(t) for t in ops[o]["outputs"] if band(t))
        P = 1
        for t in ops[o]["inputs"] + ops[o]["outputs"]:
            if an.sample[t] and not chan(t) and not band(t):
                P = max(P, p_of(t))
        return P

    def view(t, s0, s1, grad=False):
        """Rows of samples [s0, s1) of tensor t inside its resident piece."""
        if not an.sample[t]:
            return store[(n + t if grad else t, 0)]
        if chan(t):  # every block's rows, side by side (a copy: read-only use)
            r = rows_per_sample(t)
            return np.concatenate([store[(n + t if grad else t, j)][s0 * r:s1 * r] for j in range(p_of(t))], axis=-1)
        p = p_of(t)
        per = B // p
        j = s0 // per
        assert s1 <= (j + 1) * per
        r = rows_per_sample(t)
        arr = store[(n + t if grad else t, j)]
        return arr[(s0 - j * per) * r:(s1 - j * per) * r]

    bn_stats, bn_sums = {}, {}

    def channel_micro_op(it):
        """Micro-op k of an op in channel mode (D-CH): output channels block k over all
        samples.  A linear's (conv's) block k is the same op with weight rows / bias block k;
        a channel-local op (elementwise, batch norm with block k's parameters and statistics,
        max pooling, add) maps block k of its inputs to block k of its output."""
        o = ops[it.op]
        k = it.k
        out = o["outputs"][0]
        w = ts[out]["shape"][-1] // p_of(out)
        blk = slice(k * w, (k + 1) * w)
        val = dict(pval)
        sliced = set()   # parameters read as block k (their gradient is block k)
        if o["kind"] in ("linear", "conv2d"):
            x = o["inputs"][0]
            for pid in o["inputs"][1:]:
                val[pid] = pval[pid][blk]
                sliced.add(pid)
            val[x] = view(x, 0, B)
        else:
            for pid in o["inputs"]:
                if ts[pid]["kind"] == "param":
                    val[pid] = pval[pid][blk]
                    sliced.add(pid)
            if it.kind in ("F", "R"):
                for t in o["inputs"]:
                    if ts[t]["kind"] == "act":
                        val[t] = store[(t, k)]
            else:  # the backward reads block k of what the op saved
                for t in an.saved[it.op]:
                    val[t] = store[(t, k)]
        if it.kind in ("F", "R"):
            store[(out, k)][...] = net.forward_op(graph, o, val, row0=0, elem0=0, step=step)
            return
        dy = store[(n + out, k)]
        contrib = net.backward_op(graph, o, val, dy, row0=0, elem0=0, step=step)
        for tid, g in contrib.items():
            if tid in sliced:
                pgrad[tid][blk] += g
            elif ts[tid]["kind"] == "param":
                pgrad[tid] += g
            elif tid not in an.needs_grad:
                continue
            elif o["kind"] not in ("linear", "conv2d"):  # channel-local: block k of its input's gradient
                store[(n + tid, k)][...] += g
            elif chan(tid):
                r_w = g.shape[-1] // p_of(tid)
                for j in range(p_of(tid)):
                    store[(n + tid, j)][...] += g[..., j * r_w:(j + 1) * r_w]
            else:
                view(tid, 0, B, grad=True)[...] += g

    def input_pieces(x, b0, b1, grad=False):
        """(piece index, its [b0:b1] block, the slice of the whole tensor it covers) of the
        resident pieces of the window input x (band-split or unsplit)."""
        key = n + x if grad else x
        al = slice(None)
        if not band(x) and not chan(x):
            return [(0, store[(key, 0)][b0:b1], (al, al, al))]
        ax, p = (3 if chan(x) else sim.axis_of(cfg, x)), p_of(x)
        hb = ts[x]["shape"][ax] // p
        out = []
        for j in range(p):
            if (key, j) in store:
                sl = [al, al, al]
                sl[ax - 1] = slice(j * hb, (j + 1) * hb)
                out.append((j, store[(key, j)][b0:b1], tuple(sl)))
        return out

    def attr_micro_op(it):
        """Micro-op k of an op in attribute mode or of a window op reading bands (D-ATTR).
        A window op stages the input rows its output block needs (the physical merge of
        Fig. 10, padding written out: 0 for conv, -inf for max pooling), runs unpadded on
        the staged copy and, in its backward, adds the staged input gradient back into the
        pieces its rows came from.  A band-local op maps band k to band k."""
        o = ops[it.op]
        k, P = it.k, P_op(it.op)
        y = o["outputs"][0]
        val = dict(pval)
        if o["kind"] in sim.ATTR_WINDOW:
            x = o["inputs"][0]
            H, W = ts[x]["shape"][1], ts[x]["shape"][2]
            rlo, hs, clo, ws, nb = sim.staged_rect(graph, cfg, it.op, k, P)
            b0 = 0 if amode(it.op) else k * B // P
            fill = -np.inf if o["kind"] == "maxpool" else 0.0
            # the rows [rlo, rlo + hs) x columns [clo, clo + ws) of samples [b0, b0 + nb):
            # the resident pieces placed in a padded canvas, then the rectangle cut out
            pr, pc = max(0, -rlo), max(0, -clo)
            canvas = np.full((nb, H + pr + max(0, rlo + hs - H), W + pc + max(0, clo + ws - W), ts[x]["shape"][3]), fill)
            for j, blk, sl in input_pieces(x, b0, b0 + nb):
                canvas[:, pr:pr + H, pc:pc + W][(slice(None),) + sl] = blk
            xs = canvas[:, rlo + pr:rlo + pr + hs, clo + pc:clo + pc + ws].copy()
            assert (2 * n + it.op, k) in store  # the staging temporary is allocated
            store[(2 * n + it.op, k)] = xs
            o2 = dict(o, iattrs=list(o["iattrs"]))
            o2["iattrs"][1 if o["kind"] == "conv2d" else 2] = 0
            val[x] = xs
            if it.kind in ("F", "R"):
                yv = net.forward_op(graph, o2, val)
                if amode(it.op):
                    store[(y, k)][...] = yv
                else:
                    view(y, b0, b0 + nb)[...] = yv
                return
            dy = store[(n + y, k)] if amode(it.op) else view(y, b0, b0 + nb, grad=True)
            for tid, g in net.backward_op(graph, o2, val, dy).items():
                if ts[tid]["kind"] == "param":
                    pgrad[tid] += g
                elif tid in an.needs_grad:
                    store[(3 * n + it.op, k)] = g
                    canvas = np.zeros((nb, H + pr + max(0, rlo + hs - H), W + pc + max(0, clo + ws - W), g.shape[3]))
                    canvas[:, rlo + pr:rlo + pr + hs, clo + pc:clo + pc + ws] = g
                    inside = canvas[:, pr:pr + H, pc:pc + W]   # the padding's gradient is dropped
                    for j, blk, sl in input_pieces(x, b0, b0 + nb, grad=True):
                        blk[...] += inside[(slice(None),) + sl]
            return
        if it.kind in ("F", "R"):
            for t in o["inputs"]:
                if an.sample[t]:
                    val[t] = store[(t, k)]
        else:
            for t in an.saved[it.op]:
                val[t] = store[(t, k)]
        if o["kind"] == "batchnorm":  # statistics over every band (BATCH_REDUCE)
            xin, gid, bid = o["inputs"]
            eps = o["fattrs"][0]
            if it.kind == "F" and k == 0:
                bn_stats[it.op] = O.batchnorm_stats(whole(xin))
            mu, var = bn_stats[it.op]
            if it.kind in ("F", "R"):
                store[(y, k)][...] = O.batchnorm_fwd_with(val[xin], pval[gid], pval[bid], mu, var, eps)
                return
            if k == 0:
                sums = O.batchnorm_bwd_sums(whole(y, grad=True), whole(xin), pval[gid], mu, var, eps)
                bn_sums[it.op] = sums
                pgrad[gid] += sums[2]
                pgrad[bid] += sums[3]
            s1_, s2_ = bn_sums[it.op][:2]
            m = int(np.prod(ts[xin]["shape"][:-1]))
            if xin in an.needs_grad:
                store[(n + xin, k)][...] += O.batchnorm_bwd_with(
                    store[(n + y, k)], val[xin], pval[gid], mu, var, s1_, s2_, m, eps)
            return
        if it.kind in ("F", "R"):
            store[(y, k)][...] = net.forward_op(graph, o, val)
            return
        for tid, g in net.backward_op(graph, o, val, store[(n + y, k)]).items():
            if ts[tid]["kind"] == "param":
                pgrad[tid] += g
            elif tid in an.needs_grad:
                store[(n + tid, k)][...] += g

    def whole(t, grad=False):
        """All pieces of tensor t concatenated (the full batch)."""
        return np.concatenate([store[(n + t if grad else t, j)] for j in range(p_of(t))], axis=0)

    for i, it in enumerate(items):
        for pc in f_alloc.get(i, []):
            key, j = pc
            t = key - n if key >= n else key
            if key >= 2 * n:  # staging temporary: filled by the micro-op (D-ATTR)
                store[pc] = None
            elif it.kind == "SI":
                store[pc] = host.pop(pc)
            else:
                store[pc] = np.zeros(piece_shape(t), F)
        if it.kind in ("F", "R", "B") and cmode(it.op):
            channel_micro_op(it)
        elif it.kind in ("F", "R", "B") and (amode(it.op) or staged(it.op)):
            attr_micro_op(it)
        elif it.kind in ("F", "R", "B"):
            o = ops[it.op]
            P = P_op(it.op)
            s0, s1 = it.k * B // P, (it.k + 1) * B // P
            out = o["outputs"][0]
            val = dict(pval)
            reads = an.saved[it.op] if it.kind == "B" else [t for t in o["inputs"] if an.sample[t]]
            for t in reads:
                val[t] = view(t, s0, s1)
            row0 = s0 * rows_per_sample(out) if an.sample[out] else s0
            elem0 = s0 * (int(np.prod(ts[out]["shape"])) // B) if an.sample[out] else 0
            if o["kind"] == "batchnorm":
                xin, gid, bid = o["inputs"]
                eps = o["fattrs"][0]
                if it.kind == "F" and it.k == 0:
                    bn_stats[it.op] = O.batchnorm_stats(whole(xin))
                mu, var = bn_stats[it.op]
                if it.kind in ("F", "R"):
                    view(out, s0, s1)[...] = O.batchnorm_fwd_with(val[xin], pval[gid], pval[bid], mu, var, eps)
                else:
                    if it.k == 0:
                        sums = O.batchnorm_bwd_sums(whole(out, grad=True), whole(xin), pval[gid], mu, var, eps)
                        bn_sums[it.op] = sums
                        pgrad[gid] += sums[2]
                        pgrad[bid] += sums[3]
                    s1_, s2_ = bn_sums[it.op][:2]
                    m = int(np.prod(ts[xin]["shape"][:-1]))
                    if xin in an.needs_grad and ts[xin]["kind"] == "act":
                        view(xin, s0, s1, grad=True)[...] += O.batchnorm_bwd_with(
                            view(out, s0, s1, grad=True), val[xin], pval[gid], mu, var, s1_, s2_, m, eps)
            elif it.kind in ("F", "R"):
                y = net.forward_op(graph, o, val, row0=row0, elem0=elem0, step=step)
                ys = y if isinstance(y, tuple) else (y,)
                for t, yt in zip(o["outputs"], ys):
                    if an.is_loss[t]:
                        store[(t, 0)] += yt
                    elif it.kind == "F" or t == it.writes[0][0]:
                        # a replay regenerates only its target piece (other outputs may be away)
                        view(t, s0, s1)[...] = yt
            else:
                dy = None if an.is_loss[out] else view(out, s0, s1, grad=True)
                contrib = net.backward_op(graph, o, val, dy, row0=row0, elem0=elem0, step=step)
                for tid, g in contrib.items():
                    if ts[tid]["kind"] == "param":
                        pgrad[tid] += g
                    elif tid in an.needs_grad and chan(tid):  # scatter the columns into the blocks
                        r, w = rows_per_sample(tid), g.shape[1] // p_of(tid)
                        for j in range(p_of(tid)):
                            store[(n + tid, j)][s0 * r:s1 * r] += g[:, j * w:(j + 1) * w]
                    elif tid in an.needs_grad:
                        view(tid, s0, s1, grad=True)[...] += g
        elif it.kind == "SO":
            pc = it.reads[0]
            host[pc] = store[pc].copy()
        for pc in f_free.get(i, []):
            del store[pc]
    loss_id = next(o["outputs"][0] for o in ops if o["kind"] == "xent")
    loss = float(store[(loss_id, 0)][0])
    return loss, {ts[tid]["name"]: g for tid, g in pgrad.items()}
