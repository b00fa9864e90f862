"""ORACLE — test infrastructure only.

Plan-execution simulator, followed step by step from PAPER.md and the readings
DESIGN.md §4 fixes:

  schedule()  Alg. 1 (§II) with the garbled line 5 read as
              `ref_cnt -= 1` and line 6 as `== 0` (R1).
  expand()    augmented schedule (Fig. 10): op-major micro-ops
              (R10), swap-out after the last forward use / swap-in at the
              "previous computation operation", memory-centric
              recompute replay (Fig. 11), in-place re-split: a
              micro-op reads a sub-range of a coarser piece.
  Pool        best-fit over one pre-allocated slab ("best-fit memory
              allocation", "pre-allocate a large piece of GPU memory"),
              256 B alignment, lowest offset on ties, coalescing (R11).  The
              block that reaches the end of the slab is used only when no
              other block fits, so a finite slab and an unbounded one give the
              identical trace whenever the plan fits.
  simulate()  allocation only at the beginning and free only at the end of an
              operation; M_i = sum of live sizes.
"""

from __future__ import annotations

from collections import OrderedDict
from dataclasses import dataclass, field

DTYPE_BYTES = {"f32": 4, "bf16": 2, "i32": 4}
ALIGN = 256
WS_ROWS = 256
INF = 1 << 62

RESIDE, SWAP, RECOMPUTE = 0, 1, 2

# Forward tensors each backward op reads (DESIGN.md §3 table "saved").
SAVED = {
    "linear": ("in", 0),
    "relu": ("out", 0),
    "gelu": ("in", 0),
    "tanh": ("out", 0),
    "layernorm": ("in", 0),
    "add": None,
    "dropout": None,
    "softmax": ("out", 0),
    "attn_qk": ("in", 0, 1),
    "attn_pv": ("in", 0, 1),
    "embed": ("in", 0, 1),
    "cls": None,
    "xent": ("in", 0, 1),
    "conv2d": ("in", 0),
    "batchnorm": ("in", 0),
    "maxpool": ("in", 0),
    "avgpool": None,
    "flatten": None,
    "attention": (("in", 0, 1, 2), ("out", 0, 1, 2)),  # Q, K, V, C, lse, keep mask (D-SAVED)
}
AUX_OUTPUTS = {"attention": (1, 2)}  # never differentiated (same rule as net.AUX_OUTPUTS)

# Ops whose statistics span the whole batch ("the merge of
# micro-tensors can be required by the operation (e.g., batch normalization)"):
# their first forward micro-op reads every piece of the input (full-batch mean and
# variance), their first backward micro-op every piece of the input and of the
# output gradient (full-batch sums of dy and dy*xhat); the statistics live in a
# static per-op buffer, so replays and later micro-ops read only their own piece.
BATCH_REDUCE = {"batchnorm"}

# Channel (parameter-dim) split, Fig. 6 / P:L258-260, reading D-CH: a 2-D
# activation [rows, C] split along C into p contiguous blocks [rows, C/p] (the "parameter
# dim" of its producer).  Legal when its producer is a linear (micro-op k computes output
# channels block k with weight rows block k) or one of CHANNEL_EW with a channel-split
# input of the same p (micro-op k maps block k to block k), and every consumer is a linear
# reading it as X (it reads every block: the contraction over C is the merge-by-sum of
# P:L260) or one of CHANNEL_EW.  An op with a channel-split output runs in "channel mode":
# P = that p micro-ops over channel blocks, each over all samples; its other activations
# are channel-split (read whole / block k as above) or unsplit.
CHANNEL_EW = {"relu", "gelu", "tanh"}
# Images (DESIGN.md D-CH, 4-D part): an NHWC activation split along C into p blocks
# [B, H, W, C/p].  Producers: a conv2d in channel mode (micro-op k = output channels block k
# from weight rows / bias block k, over every sample; its input unsplit), or a
# CHANNEL_LOCAL4 op whose activation inputs are channel-split with the same p (ReLU, add and
# max pooling act per channel; batch norm's statistics are per channel, so block k's are
# complete within micro-op k).  Consumers: CHANNEL_LOCAL4 ops writing block k, or a conv2d
# with an unsplit or sample-split output that reads every block through a staged merge
# (D-ATTR's staging temporary, the blocks concatenated: the contraction over C needs them all).
CHANNEL_LOCAL4 = {"relu", "add", "batchnorm", "maxpool"}


def chan_local(graph, op):
    """Ops that map channel block k of their inputs to block k of their output."""
    k = op["kind"]
    return k in CHANNEL_EW or (k in CHANNEL_LOCAL4 and len(graph["tensors"][op["outputs"][0]]["shape"]) == 4)


def dim_of(cfg, t):
    c = cfg.get(t)
    return c[3] if c is not None and len(c) > 3 else 0


# Attribute (height / width) split, P:L258-260 ("split along the dim of sample, model
# parameter, or attribute (e.g., batch, channel, height, and width dimensions for images)"),
# DESIGN.md reading D-ATTR: a 4-D NHWC activation [B, H, W, C] split along H (dim 2) into p
# bands of H/p rows, piece j = rows [j H/p, (j+1) H/p) of every sample, stored [B, H/p, W, C]
# — or along W (dim 3) into p bands of W/p columns, stored [B, H, W/p, C].  An op with a
# band-split output runs in "attribute mode": micro-op k computes output band k over all
# samples.  Band-local ops (ATTR_LOCAL) read band k of band-split inputs of the same p.
# Window ops (conv2d, maxpool) read the input rows their output band needs — its own band
# plus halo rows from the neighbouring bands (or an unsplit input) — through a staged copy:
# the physical merge & split of Fig. 10, a temporary [B, Hs, Ws, C] (the rows and
# columns the output block reads, padding written out: Ws = W + 2 pad for a height band), so
# the window op runs unpadded on it; its backward scatters the staged
# input gradient back into the band pieces (overlapping halos add: merge = sum).  A
# window op whose output is not band-split reads every band of its samples the same way (a
# full merge).  Batch normalisation in band mode keeps BATCH_REDUCE's rule (its first
# micro-op reads every band: statistics over all of (N, H, W)).  The staged input of a window
# micro-op is a pool temporary allocated at the item and freed after it (key 2n + op; the
# backward's staged input gradient is key 3n + op), so the pool trace accounts for it.
ATTR_LOCAL = {"relu", "add", "batchnorm"}
ATTR_WINDOW = {"conv2d", "maxpool"}


def is_attr(graph, cfg, t):
    return dim_of(cfg, t) in (2, 3) and cfg[t][1] > 1 and graph["tensors"][t]["kind"] == "act"


def axis_of(cfg, t):
    """NHWC array axis of a band split: 1 (height, dim 2) or 2 (width, dim 3)."""
    return 1 if dim_of(cfg, t) == 2 else 2


def window_geom(op, ts, axis=1):
    """(window extent along `axis`, stride, pad) of a conv2d (R for rows, S for columns) /
    maxpool (square)."""
    if op["kind"] == "conv2d":
        return ts[op["inputs"][1]]["shape"][axis], op["iattrs"][0], op["iattrs"][1]
    return op["iattrs"][0], op["iattrs"][1], op["iattrs"][2]


def band_rows(op, ts, k, P, axis=1):
    """Input rows (axis 1; columns for axis 2) [lo, hi] (inclusive, may lie outside the
    tensor) the output band k of P of a window op reads, and the staged count hi - lo + 1."""
    R, s, pad = window_geom(op, ts, axis)
    Ho = ts[op["outputs"][0]]["shape"][axis]
    hb = Ho // P
    lo = k * hb * s - pad
    hi = ((k + 1) * hb - 1) * s - pad + R - 1
    return lo, hi, hi - lo + 1


def check_attr(graph, cfg):
    """Raise ValueError when a band (attribute) split breaks reading D-ATTR."""
    ts, ops = graph["tensors"], graph["ops"]
    producer, consumers = {}, {}
    for o in ops:
        for t in o["outputs"]:
            producer[t] = o
        for t in o["inputs"]:
            consumers.setdefault(t, []).append(o)
    for t in ts:
        tid = t["id"]
        if not is_attr(graph, cfg, tid):
            continue
        p, d = cfg[tid][1], dim_of(cfg, tid)
        if len(t["shape"]) != 4 or t["shape"][axis_of(cfg, tid)] % p:
            raise ValueError(f"tensor {tid}: a band split needs an NHWC activation whose H (W) p divides")
        same = lambda u: is_attr(graph, cfg, u) and cfg[u][1] == p and dim_of(cfg, u) == d  # noqa: E731
        po = producer[tid]
        if po["kind"] in ATTR_LOCAL:
            for x in po["inputs"]:
                if ts[x]["kind"] == "act" and not same(x):
                    raise ValueError(f"tensor {tid}: a band-local producer needs band-split inputs of the same p and dim")
        elif po["kind"] in ATTR_WINDOW:
            x = po["inputs"][0]
            if not is_attr(graph, cfg, x) and cfg[x][1] != 1:
                raise ValueError(f"tensor {tid}: its window producer's input must be unsplit or band-split")
        else:
            raise ValueError(f"tensor {tid}: producer {po['kind']} cannot write bands")
        for c in consumers.get(tid, []):
            y = c["outputs"][0]
            if c["kind"] in ATTR_LOCAL:
                if not same(y):
                    raise ValueError(f"tensor {tid}: a band-local consumer needs a band-split output of the same p and dim")
            elif c["kind"] in ATTR_WINDOW:
                if dim_of(cfg, y) == 1 and cfg[y][1] > 1:
                    raise ValueError(f"tensor {tid}: a window consumer's output cannot be channel-split")
            else:
                raise ValueError(f"tensor {tid}: consumer {c['kind']} cannot read bands")


def lag_of(cfg, t):
    """Release lag of a swapped tensor (reading D-LAG): the number of compute
    items after its swap-out before its range returns to the pool (0: at the swap-out)."""
    c = cfg.get(t)
    return c[4] if c is not None and len(c) > 4 else 0


def check_channel(graph, cfg):
    """Raise ValueError when a channel-split configuration breaks reading D-CH."""
    ts, ops = graph["tensors"], graph["ops"]
    producer, consumers = {}, {}
    for o in ops:
        for t in o["outputs"]:
            producer[t] = o
        for t in o["inputs"]:
            consumers.setdefault(t, []).append(o)

    def chan(t):
        return dim_of(cfg, t) == 1 and cfg[t][1] > 1

    for t in ts:
        tid = t["id"]
        if dim_of(cfg, tid) not in (0, 1, 2, 3):
            raise ValueError(f"tensor {tid}: split dim must be 0 (samples), 1 (channels), 2 (height) or 3 (width)")
        if not chan(tid):
            continue
        p = cfg[tid][1]
        nd = len(t["shape"])
        if t["kind"] != "act" or nd not in (2, 4) or t["shape"][-1] % p:
            raise ValueError(f"tensor {tid}: channel split needs a 2-D or NHWC activation with C % p == 0")
        po = producer[tid]
        if po["kind"] == "linear" or (po["kind"] == "conv2d" and nd == 4):
            x = po["inputs"][0]
            if not chan(x) and cfg[x][1] != 1 and ts[x]["kind"] == "act":
                raise ValueError(f"tensor {tid}: its linear's input must be unsplit or channel-split")
            if po["kind"] == "conv2d" and chan(x):
                raise ValueError(f"tensor {tid}: a channel-split conv output needs an unsplit input")
        elif chan_local(graph, po):
            for x in po["inputs"]:
                if ts[x]["kind"] == "act" and (not chan(x) or cfg[x][1] != p):
                    raise ValueError(f"tensor {tid}: an elementwise producer needs a channel-split input of the same p")
        else:
            raise ValueError(f"tensor {tid}: producer {po['kind']} cannot write channel blocks")
        for c in consumers.get(tid, []):
            y = c["outputs"][0]
            if c["kind"] == "linear" and c["inputs"][0] == tid and nd == 2:
                if not chan(y) and cfg[y][1] != 1 and ts[y]["kind"] == "act":
                    raise ValueError(f"tensor {tid}: its linear consumer's output must be unsplit or channel-split")
            elif c["kind"] == "conv2d" and nd == 4:
                if dim_of(cfg, y) != 0 and cfg[y][1] > 1:
                    raise ValueError(f"tensor {tid}: a conv reading channel blocks needs an unsplit or sample-split output")
            elif chan_local(graph, c):
                if not chan(y) or cfg[y][1] != p:
                    raise ValueError(f"tensor {tid}: an elementwise consumer needs a channel-split output of the same p")
            else:
                raise ValueError(f"tensor {tid}: consumer {c['kind']} cannot read channel blocks")


def align(n):
    return (n + ALIGN - 1) // ALIGN * ALIGN


def numel(shape):
    n = 1
    for s in shape:
        n *= s
    return n


def tbytes(t):
    return numel(t["shape"]) * DTYPE_BYTES[t["dtype"]]


def static_bytes(graph):
    """Static region: fp32 master + (bf16 copy) + fp32 grad per param, + workspace."""
    total = 0
    max1d = 1
    for t in graph["tensors"]:
        if t["kind"] != "param":
            continue
        n = numel(t["shape"])
        total += align(4 * n) + align(4 * n)
        if graph["dtype"] == "bf16":
            total += align(2 * n)
        if len(t["shape"]) == 1:
            max1d = max(max1d, n)
    bn = 0
    for o in graph["ops"]:
        if o["kind"] in BATCH_REDUCE:
            C = graph["tensors"][o["inputs"][0]]["shape"][-1]
            bn += align(16 * C)  # [mean, rstd] (forward) + [sum dy, sum dy*xhat] (backward), fp32
    return total + align(WS_ROWS * 2 * max1d * 4) + bn


def schedule(graph):
    """Alg. 1: DFS-manner topological order of the forward ops (R1)."""
    ops = graph["ops"]
    producer = {}
    for o in ops:
        for t in o["outputs"]:
            producer[t] = o["id"]
    preds = []
    succ = [[] for _ in ops]
    for o in ops:
        ps = []
        for t in o["inputs"]:
            if t in producer and producer[t] not in ps:
                ps.append(producer[t])
        preds.append(ps)
        for p in ps:
            if o["id"] not in succ[p]:
                succ[p].append(o["id"])
    for s in succ:
        s.sort()
    ref_cnt = [len(p) for p in preds]
    order = []

    def execution_scheduler(layer):
        order.append(layer)
        for nxt in succ[layer]:
            ref_cnt[nxt] -= 1
            if ref_cnt[nxt] == 0:
                execution_scheduler(nxt)

    for o in ops:
        if not preds[o["id"]]:
            execution_scheduler(o["id"])
    assert len(order) == len(ops), "graph has a cycle"
    return order


@dataclass
class Analysis:
    n: int
    producer: dict
    sample: list            # tensor id -> is a sample (splittable) tensor
    is_loss: list
    needs_grad: set
    has_bwd: list
    saved: list             # op id -> tensor ids bwd reads (non-param)
    bytes_: list
    temp: dict = field(default_factory=dict)   # staging temporary (key >= 2n, piece) -> bytes (D-ATTR)


def analyze(graph):
    ts, ops = graph["tensors"], graph["ops"]
    n = len(ts)
    producer = {}
    for o in ops:
        for t in o["outputs"]:
            producer[t] = o["id"]
    is_loss = [False] * n
    for o in ops:
        if o["kind"] == "xent":
            is_loss[o["outputs"][0]] = True
    sample = [t["kind"] != "param" and not is_loss[t["id"]] for t in ts]
    ng = {t["id"] for t in ts if t["kind"] == "param"}
    for o in ops:
        if any(i in ng for i in o["inputs"]):
            aux = AUX_OUTPUTS.get(o["kind"], ())
            ng.update(t for i, t in enumerate(o["outputs"]) if i not in aux)
    has_bwd = [o["kind"] == "xent" or any(i in ng for i in o["inputs"]) for o in ops]
    saved = []
    for o in ops:
        spec = SAVED[o["kind"]]
        lst = []
        if spec is not None:
            for part in (spec if isinstance(spec[0], tuple) else (spec,)):
                src = o["inputs"] if part[0] == "in" else o["outputs"]
                for idx in part[1:]:
                    t = src[idx]
                    if ts[t]["kind"] != "param" and t not in lst:
                        lst.append(t)
        saved.append(lst)
    return Analysis(n, producer, sample, is_loss, ng, has_bwd, saved, [tbytes(t) for t in ts])


def staged_rect(graph, cfg, o, k, P):
    """(rlo, hs, clo, ws, samples) of the staged input of micro-op k of window op o (D-ATTR):
    input rows [rlo, rlo + hs) x columns [clo, clo + ws) (padding included).  Band mode stages
    what output band k reads along the band's axis and everything along the other, for every
    sample; sample mode (a full merge) everything for B / P samples."""
    ts, op = graph["tensors"], graph["ops"][o]
    y = op["outputs"][0]
    band = is_attr(graph, cfg, y)
    span = []
    for axis in (1, 2):
        if band and axis == axis_of(cfg, y):
            lo, _, n_ = band_rows(op, ts, k, P, axis)
        else:
            lo, _, n_ = band_rows(op, ts, 0, 1, axis)
        span += [lo, n_]
    return span[0], span[1], span[2], span[3], graph["samples"] if band else graph["samples"] // P


def staged_bytes(graph, cfg, o, k, P):
    ts, op = graph["tensors"], graph["ops"][o]
    x = ts[op["inputs"][0]]
    _, hs, _, ws, nb = staged_rect(graph, cfg, o, k, P)
    return nb * hs * ws * x["shape"][3] * DTYPE_BYTES[x["dtype"]]


@dataclass
class Item:
    kind: str          # 'F' forward, 'B' backward, 'R' recompute replay, 'SO' swap-out, 'SI' swap-in
    op: int = -1
    k: int = 0
    reads: list = field(default_factory=list)    # (key, piece)
    writes: list = field(default_factory=list)
    group: int = -1    # backward group id (replays + the B item they serve)
    temps: list = field(default_factory=list)    # staging temporaries live during the item (D-ATTR)


class Pool:
    """Best-fit allocator over [base, capacity) — R11 and the tail rule above."""

    def __init__(self, base, capacity=INF):
        self.capacity = capacity
        self.free = [(base, capacity - base)]   # sorted by offset
        self.extent = base

    def alloc(self, nbytes):
        need = align(nbytes)
        best = None
        for idx, (off, ln) in enumerate(self.free):
            if off + ln == self.capacity:
                continue
            if ln >= need and (best is None or ln < self.free[best][1]):
                best = idx
        if best is None:
            idx = len(self.free) - 1
            off, ln = self.free[idx]
            if off + ln != self.capacity or ln < need:
                raise MemoryError("pool exhausted")
            best = idx
        off, ln = self.free[best]
        if ln == need:
            self.free.pop(best)
        else:
            self.free[best] = (off + need, ln - need)
        self.extent = max(self.extent, off + need)
        return off

    def release(self, off, nbytes):
        need = align(nbytes)
        i = 0
        while i < len(self.free) and self.free[i][0] < off:
            i += 1
        self.free.insert(i, (off, need))
        # coalesce with the next, then the previous block
        if i + 1 < len(self.free) and self.free[i][0] + self.free[i][1] == self.free[i + 1][0]:
            self.free[i] = (off, need + self.free[i + 1][1])
            self.free.pop(i + 1)
        if i > 0 and self.free[i - 1][0] + self.free[i - 1][1] == self.free[i][0]:
            self.free[i - 1] = (self.free[i - 1][0], self.free[i - 1][1] + self.free[i][1])
            self.free.pop(i)


def default_cfg(graph):
    return {t["id"]: (RESIDE, 1, 1) for t in graph["tensors"]}


def expand(graph, cfg, order=None, an=None, cache_bytes=0):
    """Augmented schedule: returns (items, alloc_at, free_after, fwd_end) where
    alloc_at / free_after map item index -> ordered list of (key, piece).

    cache_bytes > 0 selects the LRU-based recomputation of P:L294 (DESIGN.md reading
    D-LRU): "execute as the speed-centric manner and abandon the least recently used
    intermediate tensor once the available memory is not enough".  A regenerated piece
    stays resident for later backward groups (a later group that reads it replays
    nothing); at the end of every group the least recently used regenerated pieces
    are abandoned until the resident ones total <= cache_bytes.  cache_bytes = 0 is
    the memory-centric strategy (Fig. 11: everything regenerated per group)."""
    an = an or analyze(graph)
    order = order if order is not None else schedule(graph)
    ts, ops = graph["tensors"], graph["ops"]
    n = an.n
    an.temp = {}
    check_channel(graph, cfg)
    check_attr(graph, cfg)

    def p_of(t):
        if t >= n:
            t -= n
        if not an.sample[t] or ts[t]["kind"] != "act":
            return 1
        return cfg[t][1]

    def opt_of(t):
        return cfg[t][0]

    def P_op(o):
        if cmode(o):  # channel mode: one micro-op per channel block of the output (D-CH)
            return max(p_of(t) for t in ops[o]["outputs"] if chan(t))
        if amode(o):  # attribute mode: one micro-op per band of the output (D-ATTR)
            return max(p_of(t) for t in ops[o]["outputs"] if band(t))
        P = 1
        for t in ops[o]["inputs"] + ops[o]["outputs"]:
            if an.sample[t] and not chan(t) and not band(t):
                P = max(P, p_of(t))
        return P

    def band(t):
        if t >= n:
            t -= n
        return an.sample[t] and is_attr(graph, cfg, t)

    def amode(o):
        return any(band(t) for t in ops[o]["outputs"])

    def staged(o):
        x = ops[o]["inputs"][0]
        return ops[o]["kind"] in ATTR_WINDOW and (band(x) or amode(o) or (ops[o]["kind"] == "conv2d" and chan(x)))

    def chan(t):
        if t >= n:
            t -= n
        return an.sample[t] and ts[t]["kind"] == "act" and dim_of(cfg, t) == 1 and cfg[t][1] > 1

    def cmode(o):
        return any(chan(t) for t in ops[o]["outputs"])

    def pieces(t, k, P, o):
        """The pieces of t (or of its gradient) micro-op k of op o touches (D-CH)."""
        if t < n and not an.sample[t]:
            return [0]
        if chan(t):
            if cmode(o) and (t in ops[o]["outputs"] or chan_local(graph, ops[o])):
                return [k]
            return list(range(p_of(t)))
        if band(t):
            if ops[o]["kind"] in ATTR_WINDOW and t == ops[o]["inputs"][0]:
                # the bands holding the rows (columns) the staged input of micro-op k covers
                rlo, hs, clo, ws, _ = staged_rect(graph, cfg, o, k, P)
                ax = axis_of(cfg, t)
                lo, n_ = (rlo, hs) if ax == 1 else (clo, ws)
                H = ts[t]["shape"][ax]
                hb = H // p_of(t)
                lo, hi = max(lo, 0), min(lo + n_ - 1, H - 1)
                if lo > hi:
                    raise ValueError(f"op {o}: micro-op {k} reads no input row")
                return list(range(lo // hb, hi // hb + 1))
            return [k]
        return [k * p_of(t) // P]

    def add_temps(o, k, P, bwd):
        if not staged(o):
            return []
        nb = staged_bytes(graph, cfg, o, k, P)
        x = ops[o]["inputs"][0]
        dx = bwd and ts[x]["kind"] == "act" and x in an.needs_grad   # (the image takes no gradient)
        keys = [(2 * n + o, k)] + ([(3 * n + o, k)] if dx else [])
        for pc in keys:
            an.temp[pc] = nb
        return keys

    def ins_sample(o):
        return [t for t in ops[o]["inputs"] if an.sample[t]]

    items = []
    for o in order:
        P = P_op(o)
        for k in range(P):
            it = Item("F", o, k)
            it.reads = [(t, j) for t in ins_sample(o) for j in pieces(t, k, P, o)]
            if ops[o]["kind"] in BATCH_REDUCE and k == 0 and not cmode(o):  # (channel mode: per-block statistics)
                for t in ins_sample(o):
                    for j in range(p_of(t)):
                        if (t, j) not in it.reads:
                            it.reads.append((t, j))
            it.writes = [(t, j) for t in ops[o]["outputs"] for j in pieces(t, k, P, o)]
            it.temps = add_temps(o, k, P, False)
            items.append(it)
    fwd_end = len(items)

    def piece_nbytes(t):
        return an.bytes_[t] // p_of(t)

    cache = OrderedDict()  # regenerated pieces still resident, least recently used first
    gid = 0
    for o in reversed(order):
        if not an.has_bwd[o]:
            continue
        P = P_op(o)
        for k in range(P):
            group = []
            live_temp = set()

            def need(t, j):
                if ts[t]["kind"] != "act" or opt_of(t) != RECOMPUTE or (t, j) in live_temp:
                    return
                if (t, j) in cache:  # D-LRU hit: resident since an earlier group
                    cache.move_to_end((t, j))
                    live_temp.add((t, j))
                    return
                po = an.producer[t]
                Q = P_op(po)
                pt = p_of(t)
                for kk in range(j * Q // pt, (j + 1) * Q // pt):
                    for u in ins_sample(po):
                        for jj in pieces(u, kk, Q, po):
                            need(u, jj)
                    r = Item("R", po, kk, group=gid)
                    r.reads = [(u, jj) for u in ins_sample(po) for jj in pieces(u, kk, Q, po)]
                    r.writes = [(t, j)]
                    r.temps = add_temps(po, kk, Q, False)
                    group.append(r)
                live_temp.add((t, j))
                cache[(t, j)] = piece_nbytes(t)

            saved_pieces = [(t, j) for t in an.saved[o] for j in pieces(t, k, P, o)]
            if ops[o]["kind"] in BATCH_REDUCE and k == 0 and not cmode(o):
                for t in an.saved[o]:
                    for j in range(p_of(t)):
                        if (t, j) not in saved_pieces:
                            saved_pieces.append((t, j))
            for (t, j) in saved_pieces:
                need(t, j)
            b = Item("B", o, k, group=gid)
            b.temps = add_temps(o, k, P, True)
            b.reads = list(saved_pieces)
            for t in ops[o]["outputs"]:
                if not an.is_loss[t] and t in an.needs_grad:
                    for j in pieces(t, k, P, o):
                        b.reads.append((n + t, j))
                    if ops[o]["kind"] in BATCH_REDUCE and k == 0 and not cmode(o):
                        for j in range(p_of(t)):
                            if (n + t, j) not in b.reads:
                                b.reads.append((n + t, j))
            for t in ops[o]["inputs"]:
                if ts[t]["kind"] == "act" and t in an.needs_grad:
                    for j in pieces(t, k, P, o):
                        w = (n + t, j)
                        if w not in b.writes:
                            b.writes.append(w)
            group.append(b)
            items.extend(group)
            gid += 1
            # abandon least recently used regenerated pieces beyond the cache limit
            while cache and sum(cache.values()) > cache_bytes:
                cache.popitem(last=False)

    # ---- lifetimes -------------------------------------------------------------
    touches = {}
    for i, it in enumerate(items):
        for pc in it.writes + it.reads:
            touches.setdefault(pc, []).append(i)

    def cls(key):
        if key >= n:
            return "grad"
        t = ts[key]
        if t["kind"] in ("input", "label"):
            return "input"
        if an.is_loss[key]:
            return "loss"
        return "act"

    alloc_at, free_after = {}, {}
    swap_out_after = {}       # forward item index -> [pieces]
    swap_in_before = {}       # pre-insertion item index -> [pieces]
    lag_free = {}             # pre-insertion item index -> [swapped-out pieces freed after it]
    temp_spans = []
    for pc, idxs in touches.items():
        key, j = pc
        c = cls(key)
        if c == "input":
            free_after.setdefault(max(idxs), []).append(pc)
            continue
        if c == "loss":
            alloc_at.setdefault(min(idxs), []).append(pc)
            continue
        if c == "grad":
            alloc_at.setdefault(min(idxs), []).append(pc)
            free_after.setdefault(max(idxs), []).append(pc)
            continue
        fw = [i for i in idxs if i < fwd_end]
        bw = [i for i in idxs if i >= fwd_end]
        opt = opt_of(key)
        alloc_at.setdefault(min(fw), []).append(pc)
        if not bw or opt == RESIDE:
            free_after.setdefault(max(idxs), []).append(pc)
        elif opt == SWAP:
            swap_out_after.setdefault(max(fw), []).append(pc)
            lead = max(1, cfg[key][2])
            pos = max(min(bw) - lead, fwd_end)
            swap_in_before.setdefault(pos, []).append(pc)
            free_after.setdefault(max(bw), []).append(pc)
            # D-LAG: the range the swap-out frees returns to the pool only after the
            # lag-th compute item behind it (the copy's time), and before the swap-in
            q = min(max(fw) + lag_of(cfg, key), pos - 1)
            if lag_of(cfg, key) > 0 and q > max(fw):
                lag_free.setdefault(q, []).append(pc)
        else:  # RECOMPUTE: forward lifetime, then one residency per regeneration
            free_after.setdefault(max(fw), []).append(pc)
            # a residency starts at the replay writing the piece and ends at its last
            # touch before the next replay of it (memory-centric: one per group)
            # (a regeneration may be several replays of one group, when the producer has
            # more micro-ops than the piece: the group's first one starts the residency)
            seen, starts = set(), []
            for i in bw:
                if items[i].kind == "R" and pc in items[i].writes and items[i].group not in seen:
                    seen.add(items[i].group)
                    starts.append(i)
            for a, st in enumerate(starts):
                end = starts[a + 1] if a + 1 < len(starts) else None
                span = [i for i in bw if i >= st and (end is None or i < end)]
                alloc_at.setdefault(st, []).append(pc)
                free_after.setdefault(max(span), []).append(pc)
                temp_spans.append((pc, st, max(span)))

    # ---- final item list with SO / SI items -----------------------------------
    final = []
    f_alloc, f_free = {}, {}
    for i, it in enumerate(items):
        for pc in sorted(swap_in_before.get(i, [])):
            si = Item("SI")
            si.writes = [pc]
            f_alloc[len(final)] = [pc]
            final.append(si)
        idx = len(final)
        final.append(it)
        # allocation order: the item's write order, then its reads (temps never
        # appear as reads before a write; inputs are allocated at start)
        allocs = alloc_at.get(i, [])
        ordered = [pc for pc in it.writes if pc in allocs] + [pc for pc in it.reads if pc in allocs and pc not in it.writes]
        assert len(ordered) == len(set(allocs)), (it, allocs)
        ordered += it.temps  # staging temporaries last (D-ATTR)
        if ordered:
            f_alloc[idx] = ordered
        if i in free_after or i in lag_free or it.temps:
            f_free[idx] = sorted(free_after.get(i, []) + lag_free.get(i, []) + it.temps)
        for pc in sorted(swap_out_after.get(i, [])):
            so = Item("SO")
            so.reads = [pc]
            if not any(pc in v for v in lag_free.values()):
                f_free[len(final)] = [pc]
            final.append(so)
    return final, f_alloc, f_free, fwd_end, an


@dataclass
class SimResult:
    items: list
    trace: list            # (seq, item, 'A'|'F', key, piece, offset, bytes)
    static: int
    peak_live: int
    peak_extent: int
    live_after_alloc: list  # per item, dynamic live bytes
    n_replay: int
    d2h_bytes: int
    h2d_bytes: int


def simulate(graph, cfg=None, order=None, capacity=INF, cache_bytes=0):
    cfg = cfg or default_cfg(graph)
    items, f_alloc, f_free, fwd_end, an = expand(graph, cfg, order, cache_bytes=cache_bytes)
    ts = graph["tensors"]
    n = an.n
    base = static_bytes(graph)
    pool = Pool(base, capacity)

    def pbytes(pc):
        key, j = pc
        if key >= 2 * n:
            return an.temp[pc]
        t = key - n if key >= n else key
        if not an.sample[t] or ts[t]["kind"] != "act":
            return an.bytes_[t]
        return an.bytes_[t] // cfg[t][1]

    where = {}
    trace = []
    live = 0
    peak = 0
    lal = []

    def do_alloc(item_idx, pc):
        nonlocal live
        b = pbytes(pc)
        off = pool.alloc(b)
        assert pc not in where, ("double alloc", pc)
        where[pc] = off
        live += align(b)
        trace.append((len(trace), item_idx, "A", pc[0], pc[1], off, b))

    def do_free(item_idx, pc):
        nonlocal live
        b = pbytes(pc)
        off = where.pop(pc)
        pool.release(off, b)
        live -= align(b)
        trace.append((len(trace), item_idx, "F", pc[0], pc[1], off, b))

    for t in ts:
        if t["kind"] in ("input", "label"):
            do_alloc(-1, (t["id"], 0))
    peak = live
    d2h = h2d = nrep = 0
    for i, it in enumerate(items):
        for pc in f_alloc.get(i, []):
            do_alloc(i, pc)
        for pc in it.reads:
            assert pc in where, ("read of non-resident piece", i, it, pc)
        for pc in it.writes:
            assert pc in where, ("write to unallocated piece", i, it, pc)
        lal.append(live)
        peak = max(peak, live)
        if it.kind == "SO":
            d2h += pbytes(it.reads[0])
        elif it.kind == "SI":
            h2d += pbytes(it.writes[0])
        elif it.kind == "R":
            nrep += 1
        for pc in f_free.get(i, []):
            do_free(i, pc)
    for pc in sorted(list(where.keys())):
        do_free(len(items), pc)
    return SimResult(items, trace, base, base + peak, pool.extent, lal, nrep, d2h, h2d)
