"""Stock-PyTorch runtime of an exported TSPLIT augmented graph.

PAPER.md §VI-D: "we could convert TSPLIT augmented dataflow graph into
PyTorch ... After adding the extra split/swap/regenerate operators in existing
frameworks, the augmented dataflow graph of TSPLIT can be converted into the executable
model in PyTorch".  `export.export_torch` writes a standalone Python module: this file's
source (it imports only torch), the graph, the plan's augmented item list and its
allocation trace as literals, and an `AugmentedStep` class that executes them with stock
torch operators — split micro-ops on views of their pieces, swap-out / swap-in as copies
to pinned host tensors on side streams (event-ordered), recompute replays as
re-executed forward micro-ops, frees as dropped references.  No libtsplit, no custom
kernels: it is the paper's "other frameworks" path, not the hot path (which is the C-ABI
library).  Backward micro-ops use torch.autograd on the re-executed micro-op where the op
saves its inputs, and the closed forms where it saves its output (relu, tanh, softmax)
or needs whole-batch terms (batch normalisation, R13).

Semantics restated from the paper / DESIGN.md readings (this runtime shares no code with
the oracle or the CUDA path): R14 loss = mean over the graph's batch; R15 / D-RNG dropout
keep decisions from Philox4x32-10; R16 erf-GELU, LayerNorm eps from the op, first-max
max-pool routing; R13 batch statistics over every piece; D-SAVED the tensors each
backward reads.
"""

import math

import torch
import torch.nn.functional as Fn

# ----------------------------------------------------------------- Philox (D-RNG)
_M0, _M1 = 0xD2511F53, 0xCD9E8D57
_W0, _W1 = 0x9E3779B9, 0xBB67AE85
_KEY1 = 0x5453504C
_M32 = 0xFFFFFFFF


def _philox_words(ctr, seed, step):
    """Philox4x32-10 of counters (ctr lo, ctr hi, step, 0) under key (seed, 0x5453504C);
    int64 tensors holding 32-bit values (products wrap modulo 2^64, the bits kept)."""
    c0 = ctr & _M32
    c1 = (ctr >> 32) & _M32
    c2 = torch.full_like(c0, step & _M32)
    c3 = torch.zeros_like(c0)
    k0, k1 = seed & _M32, _KEY1
    for _ in range(10):
        p0 = c0 * _M0
        p1 = c2 * _M1
        hi0, lo0 = (p0 >> 32) & _M32, p0 & _M32
        hi1, lo1 = (p1 >> 32) & _M32, p1 & _M32
        c0, c1, c2, c3 = hi1 ^ c1 ^ k0, lo1, hi0 ^ c3 ^ k1, lo0
        k0 = (k0 + _W0) & _M32
        k1 = (k1 + _W1) & _M32
    return torch.stack([c0, c1, c2, c3])


def dropout_keep(shape, elem0, p, seed, step, device):
    """Keep decisions of elements elem0 .. elem0 + numel of a tensor (global element
    index): element i draws the 16-bit half (i & 1) of word (i >> 1) & 3 of the Philox
    call of counter i >> 3; keep = draw >= floor(p 2^16)."""
    n = math.prod(shape)
    idx = torch.arange(elem0, elem0 + n, dtype=torch.int64, device=device)
    words = _philox_words(idx >> 3, seed, step)
    w = torch.gather(words, 0, ((idx >> 1) & 3).unsqueeze(0))[0]
    half = (w >> (16 * (idx & 1))) & 0xFFFF
    thr = min(int(math.floor(p * 65536.0)), 65535)
    return (half >= thr).reshape(shape)


def pack_mask_words(keep):
    """[..., s] bool -> [..., ceil(s/32)] int32 words, key 32w + j at bit j."""
    s = keep.shape[-1]
    nw = (s + 31) // 32
    pad = torch.zeros(keep.shape[:-1] + (nw * 32 - s,), dtype=torch.bool, device=keep.device)
    bits = torch.cat([keep, pad], -1).reshape(keep.shape[:-1] + (nw, 32)).to(torch.int64)
    w = (bits << torch.arange(32, device=keep.device, dtype=torch.int64)).sum(-1)
    return ((w + 2 ** 31) % 2 ** 32 - 2 ** 31).to(torch.int32)


def unpack_mask_words(words, s):
    w = words.to(torch.int64) & _M32
    bits = (w.unsqueeze(-1) >> torch.arange(32, device=words.device, dtype=torch.int64)) & 1
    return bits.reshape(words.shape[:-1] + (words.shape[-1] * 32,))[..., :s].bool()


# ----------------------------------------------------------------- operators
def _heads(x, heads, seq):
    nb = x.shape[0] // seq
    return x.reshape(nb, seq, heads, -1).permute(0, 2, 1, 3)


def _merge(xh):
    nb, a, s, d = xh.shape
    return xh.permute(0, 2, 1, 3).reshape(nb * s, a * d)


def gelu(x):
    return 0.5 * x * (1.0 + torch.erf(x / math.sqrt(2.0)))


def layernorm(x, g, b, eps):
    mu = x.mean(-1, keepdim=True)
    var = ((x - mu) ** 2).mean(-1, keepdim=True)
    return (x - mu) / torch.sqrt(var + eps) * g + b


def attention(q, k, v, heads, seq, alpha, p, seed, elem0, step, keep=None):
    """C = dropout(softmax(alpha Q_h K_h^T)) V_h (heads merged), lse, keep mask."""
    s = alpha * (_heads(q, heads, seq) @ _heads(k, heads, seq).transpose(-1, -2))
    lse = torch.logsumexp(s, -1)
    pr = torch.softmax(s, -1)
    if keep is None:
        keep = (torch.ones(s.shape, dtype=torch.bool, device=s.device) if p == 0.0
                else dropout_keep(tuple(s.shape), elem0, p, seed, step, s.device))
    pd = torch.where(keep, pr / (1.0 - p), torch.zeros_like(pr)) if p > 0.0 else pr
    return _merge(pd @ _heads(v, heads, seq)), lse, keep


def conv2d(x, w, b, stride, pad):
    y = Fn.conv2d(x.permute(0, 3, 1, 2), w.permute(0, 3, 1, 2), b, stride=stride, padding=pad)
    return y.permute(0, 2, 3, 1)


def _windows(x, k, stride, pad, fill):
    """NHWC windows of x: list over (r, s) of [N,P,Q,C] slices of the padded input."""
    N, H, W, C = x.shape
    P = (H + 2 * pad - k) // stride + 1
    Q = (W + 2 * pad - k) // stride + 1
    xp = Fn.pad(x, (0, 0, pad, pad, pad, pad), value=fill)
    return [xp[:, r:r + stride * P:stride, s:s + stride * Q:stride, :] for r in range(k) for s in range(k)], xp, P, Q


def maxpool(x, k, stride, pad):
    wins, _, _, _ = _windows(x, k, stride, pad, float("-inf"))
    y = wins[0]
    for w in wins[1:]:
        y = torch.maximum(y, w)
    return y


def maxpool_bwd(dy, x, k, stride, pad):
    """Gradient to the first maximum of each window in row-major order (R16)."""
    wins, xp, P, Q = _windows(x, k, stride, pad, float("-inf"))
    y = maxpool(x, k, stride, pad)
    taken = torch.zeros(dy.shape, dtype=torch.bool, device=dy.device)
    dxp = torch.zeros(xp.shape, dtype=dy.dtype, device=dy.device)
    i = 0
    for r in range(k):
        for s in range(k):
            hit = (wins[i] == y) & ~taken
            dxp[:, r:r + stride * P:stride, s:s + stride * Q:stride, :] += torch.where(hit, dy, torch.zeros_like(dy))
            taken |= hit
            i += 1
    H, W = x.shape[1], x.shape[2]
    return dxp[:, pad:pad + H, pad:pad + W, :]


def xent(z, labels, b_global):
    return (torch.logsumexp(z, 1) - z.gather(1, labels.long().unsqueeze(1))[:, 0]).sum() / b_global


AUX_OUTPUTS = {"attention": (1, 2)}


class Runtime:
    """Executes ITEMS (kind, op, k, aux) with ALLOC / FREE (per item: [(key, piece)]) of a
    graph SPEC under CFG {tensor id: (opt, p_num, lead, dim)}."""

    def __init__(self, spec, cfg, items, allocs, frees, device, dtype):
        self.spec, self.cfg, self.items, self.allocs, self.frees = spec, cfg, items, allocs, frees
        self.device, self.dtype = torch.device(device), dtype
        self.ts, self.ops = spec["tensors"], spec["ops"]
        self.n, self.B = len(self.ts), spec["samples"]
        # every non-parameter tensor except the loss carries the sample (split) leading dim
        loss_ids = {o["outputs"][0] for o in self.ops if o["kind"] == "xent"}
        self.sample = {t["id"]: t["kind"] != "param" and t["id"] not in loss_ids for t in self.ts}
        self.loss_id = next(iter(loss_ids))
        self.needs_grad = {t["id"] for t in self.ts if t["kind"] == "param"}
        for o in self.ops:
            if any(i in self.needs_grad for i in o["inputs"]):
                aux = AUX_OUTPUTS.get(o["kind"], ())
                self.needs_grad.update(t for j, t in enumerate(o["outputs"]) if j not in aux)
        self.cuda = self.device.type == "cuda"
        if self.cuda:
            self.s_d2h, self.s_h2d = torch.cuda.Stream(self.device), torch.cuda.Stream(self.device)

    # -- layout ---------------------------------------------------------------
    def p_of(self, t):
        return self.cfg[t][1] if (self.sample[t] and self.ts[t]["kind"] == "act") else 1

    # split dims (DESIGN.md D-CH, D-ATTR): 0 samples, 1 channels (last axis), 2 / 3 height / width bands
    def dim(self, t):
        c = self.cfg[t]
        return c[3] if len(c) > 3 and c[1] > 1 and self.sample[t] and self.ts[t]["kind"] == "act" else 0

    def chan(self, t):
        return self.dim(t) == 1

    def band(self, t):
        return self.dim(t) in (2, 3)

    def axis(self, t):  # NHWC array axis of a band split
        return 1 if self.dim(t) == 2 else 2

    def cmode(self, o):  # channel mode: micro-op k = channel block k of the output, every sample
        return any(self.chan(t) for t in self.ops[o]["outputs"])

    def amode(self, o):  # attribute mode: micro-op k = band k of the output, every sample
        return any(self.band(t) for t in self.ops[o]["outputs"])

    def staged(self, o):  # a window op reading its input through a staged rectangle
        op = self.ops[o]
        x = op["inputs"][0]
        return op["kind"] in ("conv2d", "maxpool") and (
            self.band(x) or self.amode(o) or (op["kind"] == "conv2d" and self.chan(x)))

    def P_op(self, o):
        outs = self.ops[o]["outputs"]
        if self.cmode(o):
            return max(self.p_of(t) for t in outs if self.chan(t))
        if self.amode(o):
            return max(self.p_of(t) for t in outs if self.band(t))
        P = 1
        for t in self.ops[o]["inputs"] + outs:
            if self.sample[t] and not self.chan(t) and not self.band(t):
                P = max(P, self.p_of(t))
        return P

    def rows(self, t):
        return self.ts[t]["shape"][0] // self.B

    def piece_shape(self, t):
        sh = list(self.ts[t]["shape"])
        if self.chan(t):
            sh[-1] //= self.p_of(t)
        elif self.band(t):
            sh[self.axis(t)] //= self.p_of(t)
        elif self.sample[t]:
            sh[0] //= self.p_of(t)
        return sh

    def tdtype(self, t):
        return {"i32": torch.int32, "f32": self.dtype if self.dtype == torch.float64 else torch.float32,
                "bf16": self.dtype}[self.ts[t]["dtype"]]

    def view(self, t, s0, s1, grad=False):
        key = self.n + t if grad else t
        if not self.sample[t]:
            return self.store[(key, 0)]
        per = self.B // self.p_of(t)
        j = s0 // per
        r = self.rows(t)
        return self.store[(key, j)][(s0 - j * per) * r:(s1 - j * per) * r]

    def whole(self, t, grad=False):
        key = self.n + t if grad else t
        return torch.cat([self.store[(key, j)] for j in range(self.p_of(t))], 0)

    def c(self, x):  # compute precision
        return x.to(torch.float64 if self.dtype == torch.float64 else torch.float32)

    # -- one step -------------------------------------------------------------
    def run(self, params, inputs, step=0):
        dev = self.device
        self.pval = {t["id"]: self.c(torch.as_tensor(params[t["name"]]).to(dev)) for t in self.ts if t["kind"] == "param"}
        self.pgrad = {k: torch.zeros_like(v) for k, v in self.pval.items()}
        self.store, self.host, self.ev = {}, {}, {}
        self.bn = {}
        for t in self.ts:
            if t["kind"] in ("input", "label"):
                a = torch.as_tensor(inputs[t["name"]]).to(dev)
                self.store[(t["id"], 0)] = a.to(self.tdtype(t["id"])) if t["dtype"] != "i32" else a
        with torch.no_grad():
            for i, (kind, op, k, aux) in enumerate(self.items):
                for key, j in self.allocs[i]:
                    t = key - self.n if key >= self.n else key
                    if key >= 2 * self.n:  # a staging temporary (D-ATTR): torch allocates its own
                        self.store[(key, j)] = None
                    elif kind == "SI":
                        self._swap_in(key, j)
                    else:
                        self.store[(key, j)] = torch.zeros(self.piece_shape(t), dtype=self.tdtype(t), device=dev)
                special = kind in ("F", "R", "B") and (self.cmode(op) or self.amode(op) or self.staged(op) or any(
                    self.chan(t) for t in self.ops[op]["inputs"]))
                if special:
                    self._split_micro_op(op, k, kind, step)
                elif kind in ("F", "R"):
                    self._forward(op, k, kind == "R", step)
                elif kind == "B":
                    self._backward(op, k, step)
                elif kind == "SO":
                    self._swap_out(aux >> 16, aux & 0xFFFF)
                for key, j in self.frees[i]:
                    del self.store[(key, j)]
        loss = float(self.store.get((self.loss_id, 0), torch.zeros(1))[0])
        return loss, {self.ts[t]["name"]: g for t, g in self.pgrad.items()}

    def _swap_out(self, key, j):
        x = self.store[(key, j)]
        if self.cuda:
            h = torch.empty(x.shape, dtype=x.dtype, pin_memory=True)
            ev = torch.cuda.Event()
            ev.record(torch.cuda.current_stream(self.device))
            with torch.cuda.stream(self.s_d2h):
                self.s_d2h.wait_event(ev)
                h.copy_(x, non_blocking=True)
                x.record_stream(self.s_d2h)
                done = torch.cuda.Event()
                done.record(self.s_d2h)
            self.ev[(key, j)] = done
            self.host[(key, j)] = h
        else:
            self.host[(key, j)] = x.clone()

    def _swap_in(self, key, j):
        h = self.host.pop((key, j))
        if self.cuda:
            with torch.cuda.stream(self.s_h2d):
                self.s_h2d.wait_event(self.ev.pop((key, j)))
                x = h.to(self.device, non_blocking=True)
                done = torch.cuda.Event()
                done.record(self.s_h2d)
            torch.cuda.current_stream(self.device).wait_event(done)
            x.record_stream(torch.cuda.current_stream(self.device))
            self.store[(key, j)] = x
        else:
            self.store[(key, j)] = h

    def _offsets(self, op, s0):
        o = self.ops[op]
        out = o["outputs"][0]
        row0 = s0 * self.rows(out) if self.sample[out] else s0
        elem0 = s0 * (math.prod(self.ts[out]["shape"]) // self.B) if self.sample[out] else 0
        return row0, elem0

    def _forward(self, op, k, replay, step):
        o = self.ops[op]
        kd, ia, fa = o["kind"], o["iattrs"], o["fattrs"]
        P = self.P_op(op)
        s0, s1 = k * self.B // P, (k + 1) * self.B // P
        row0, elem0 = self._offsets(op, s0)
        ins = [self.pval[t] if t in self.pval else (self.view(t, s0, s1) if self.sample[t] else self.store[(t, 0)])
               for t in o["inputs"]]
        x = [self.c(a) if a.dtype.is_floating_point else a for a in ins]
        outs = o["outputs"]
        if kd == "batchnorm":
            if k == 0 and not replay:
                xa = self.c(self.whole(o["inputs"][0]))
                ax = tuple(range(xa.dim() - 1))
                mu = xa.mean(ax)
                self.bn[op] = (mu, ((xa - mu) ** 2).mean(ax))
            mu, var = self.bn[op]
            ys = [(x[0] - mu) / torch.sqrt(var + fa[0]) * x[1] + x[2]]
        elif kd == "attention":
            b0 = s0
            c, lse, keep = attention(x[0], x[1], x[2], ia[0], ia[1], fa[0], fa[1], ia[2],
                                     b0 * ia[0] * ia[1] * ia[1], step)
            ys = [c, lse, pack_mask_words(keep)]
        elif kd == "xent":
            self.store[(outs[0], 0)] += xent(x[0], x[1], self.B)
            return
        else:
            ys = [self._fwd_op(kd, x, ia, fa, row0, elem0, step)]
        for j, (t, y) in enumerate(zip(outs, ys)):
            if replay and not self._replay_target(t, s0):
                continue
            self.view(t, s0, s1).copy_(y)

    def _replay_target(self, t, s0):
        # a replay regenerates only the piece it was issued for (others may be swapped away)
        if not self.sample[t]:
            return (t, 0) in self.store
        return (t, s0 // (self.B // self.p_of(t))) in self.store

    def _fwd_op(self, kd, x, ia, fa, row0, elem0, step):
        if kd == "linear":
            return x[0] @ x[1].T + x[2]
        if kd == "relu":
            return torch.clamp_min(x[0], 0.0)
        if kd == "gelu":
            return gelu(x[0])
        if kd == "tanh":
            return torch.tanh(x[0])
        if kd == "layernorm":
            return layernorm(x[0], x[1], x[2], fa[0])
        if kd == "add":
            return x[0] + x[1]
        if kd == "dropout":
            if fa[0] == 0.0:
                return x[0]
            keep = dropout_keep(tuple(x[0].shape), elem0, fa[0], ia[0], step, x[0].device)
            return torch.where(keep, x[0] / (1.0 - fa[0]), torch.zeros_like(x[0]))
        if kd == "softmax":
            if ia and ia[0]:  # causal: keys j > query i dropped
                s = x[0].shape[-1]
                mask = torch.triu(torch.ones(s, s, dtype=torch.bool, device=x[0].device), 1)
                return torch.softmax(x[0].masked_fill(mask, float("-inf")), -1)
            return torch.softmax(x[0], -1)
        if kd == "attn_qk":
            return fa[0] * (_heads(x[0], ia[0], ia[1]) @ _heads(x[1], ia[0], ia[1]).transpose(-1, -2))
        if kd == "attn_pv":
            return _merge(x[0] @ _heads(x[1], ia[0], ia[1]))
        if kd == "embed":
            pos = torch.arange(row0, row0 + x[0].shape[0], device=x[0].device) % ia[0]
            return x[2][x[0].long()] + x[3][pos] + x[4][x[1].long()]
        if kd == "cls":
            return x[0][::ia[0]]
        if kd == "conv2d":
            return conv2d(x[0], x[1], x[2] if len(x) > 2 else None, ia[0], ia[1])
        if kd == "maxpool":
            return maxpool(x[0], ia[0], ia[1], ia[2])
        if kd == "avgpool":
            return x[0].mean((1, 2))
        if kd == "flatten":
            return x[0].reshape(x[0].shape[0], -1)
        raise NotImplementedError(kd)

    # -- channel (D-CH) and band (D-ATTR) micro-ops -------------------------------
    def _rect(self, o, k, P):
        """(rlo, hs, clo, ws, samples) of the input rectangle micro-op k of window op o reads
        (padding included): what output band k needs along the band's axis, all else."""
        op, ts = self.ops[o], self.ts
        y = op["outputs"][0]
        band = self.band(y)
        span = []
        for ax in (1, 2):
            if op["kind"] == "conv2d":
                R, s, pad = ts[op["inputs"][1]]["shape"][ax], op["iattrs"][0], op["iattrs"][1]
            else:
                R, s, pad = op["iattrs"][0], op["iattrs"][1], op["iattrs"][2]
            here = band and self.axis(y) == ax
            hb = ts[y]["shape"][ax] // P if here else ts[y]["shape"][ax]
            kk = k if here else 0
            lo = kk * hb * s - pad
            span += [lo, ((kk + 1) * hb - 1) * s - pad + R - lo]
        return span[0], span[1], span[2], span[3], (self.B if band else self.B // P)

    def _pieces(self, t, b0, b1, grad=False):
        """(rows of samples [b0, b1) of each resident piece of t, its index tuple into the
        whole tensor's rows of those samples) — channel blocks, bands, or the unsplit tensor."""
        key, al, r = (self.n + t if grad else t), slice(None), self.rows(t)
        nd = len(self.ts[t]["shape"])
        if not (self.chan(t) or self.band(t)):
            return [(self.store[(key, 0)][b0 * r:b1 * r], (al,) * nd)]
        ax = nd - 1 if self.chan(t) else self.axis(t)
        w = self.ts[t]["shape"][ax] // self.p_of(t)
        out = []
        for j in range(self.p_of(t)):
            if (key, j) in self.store:
                sl = [al] * nd
                sl[ax] = slice(j * w, (j + 1) * w)
                out.append((self.store[(key, j)][b0 * r:b1 * r], tuple(sl)))
        return out

    def _gather(self, t, b0, nb, rlo, hs, clo, ws, fill):
        """The staged rectangle of t: rows [rlo, rlo + hs) x columns [clo, clo + ws) of samples
        [b0, b0 + nb), fill outside t (the physical merge of Fig. 10)."""
        H, W, C = self.ts[t]["shape"][1:]
        pr, pc = max(0, -rlo), max(0, -clo)
        cv = torch.full((nb, H + pr + max(0, rlo + hs - H), W + pc + max(0, clo + ws - W), C), fill,
                        dtype=torch.float64 if self.dtype == torch.float64 else torch.float32, device=self.device)
        inner = cv[:, pr:pr + H, pc:pc + W]
        for blk, sl in self._pieces(t, b0, b0 + nb):
            inner[sl] = self.c(blk)
        return cv[:, rlo + pr:rlo + pr + hs, clo + pc:clo + pc + ws]

    def _scatter(self, t, b0, nb, rlo, hs, clo, ws, g):
        """Add the staged rectangle's gradient g into t's gradient pieces (padding dropped)."""
        H, W, C = self.ts[t]["shape"][1:]
        pr, pc = max(0, -rlo), max(0, -clo)
        cv = torch.zeros((nb, H + pr + max(0, rlo + hs - H), W + pc + max(0, clo + ws - W), C), dtype=g.dtype,
                         device=g.device)
        cv[:, rlo + pr:rlo + pr + hs, clo + pc:clo + pc + ws] = g
        inner = cv[:, pr:pr + H, pc:pc + W]
        for blk, sl in self._pieces(t, b0, b0 + nb, grad=True):
            blk.copy_((self.c(blk) + inner[sl]).to(blk.dtype))

    def _split_micro_op(self, op, k, kind, step):
        """Micro-op k of an op in channel mode (output channels block k: a linear's / conv's
        weight rows and bias block k, a channel-local op's block k), in attribute mode (output
        band k) or of a window op reading bands or channel blocks through a staged rectangle."""
        o = self.ops[op]
        kd, ia, fa = o["kind"], list(o["iattrs"]), o["fattrs"]
        P = self.P_op(op)
        ins, out = o["inputs"], o["outputs"][0]
        cm, am, st = self.cmode(op), self.amode(op), self.staged(op)
        w = self.ts[out]["shape"][-1] // self.p_of(out) if cm else None
        blk = slice(k * w, (k + 1) * w) if cm else None
        b0 = 0 if (cm or am) else k * self.B // P
        nb = self.B if (cm or am) else self.B // P
        rect = self._rect(op, k, P) if st else None
        x, sliced = [], set()
        for i, t in enumerate(ins):
            if t in self.pval:
                sliced_here = cm and (kd in ("linear", "conv2d") or kd == "batchnorm")
                x.append(self.pval[t][blk] if sliced_here else self.pval[t])
                if sliced_here:
                    sliced.add(t)
            elif st and i == 0:
                x.append(self._gather(t, b0, nb, rect[0], rect[1], rect[2], rect[3],
                                      float("-inf") if kd == "maxpool" else 0.0))
            elif (cm or am) and (self.chan(t) or self.band(t)) and kd not in ("linear", "conv2d"):
                v = self.store.get((t, k))   # (a backward reads only what its op saved)
                x.append(None if v is None else self.c(v))
            elif self.chan(t):  # a linear / conv reading every block: merged along the channels
                x.append(torch.cat([self.c(b) for b, _ in self._pieces(t, b0, b0 + nb)], -1))
            else:
                v = self.store[(t, 0)]
                x.append(self.c(v) if v.dtype.is_floating_point else v)
        if st:  # the window op runs unpadded on the staged rectangle
            ia[1 if kd == "conv2d" else 2] = 0

        def bn_stats():
            xa = self.c(self.whole(ins[0]))
            ax = tuple(range(xa.dim() - 1))
            mu = xa.mean(ax)
            self.bn[op] = (mu, ((xa - mu) ** 2).mean(ax))

        def evaluate(xs):
            if kd == "batchnorm":
                if cm:  # block k holds every sample of its channels: its own statistics
                    mu = xs[0].mean((0, 1, 2))
                    var = ((xs[0] - mu) ** 2).mean((0, 1, 2))
                else:
                    mu, var = self.bn[op]
                return (xs[0] - mu) / torch.sqrt(var + fa[0]) * xs[1] + xs[2]
            return self._fwd_op(kd, xs, ia, fa, 0, 0, step)

        if kind in ("F", "R"):
            if kd == "batchnorm" and am and k == 0 and kind == "F":
                bn_stats()
            y = evaluate(x)
            if cm or am:
                if (out, k) in self.store:  # (a replay regenerates only its own piece)
                    self.store[(out, k)].copy_(y)
            else:
                self.view(out, b0, b0 + nb).copy_(y)
            return
        dy = self.c(self.store[(self.n + out, k)] if (cm or am) else self.view(out, b0, b0 + nb, grad=True))
        if kd == "batchnorm" and am:  # statistics over every band: the sums of all of dY and X (R13)
            xin, gid, bid = ins
            mu, var = self.bn[op]
            rstd = 1.0 / torch.sqrt(var + fa[0])
            g = self.pval[gid]
            if k == 0:
                dya, xa = self.c(self.whole(out, grad=True)), self.c(self.whole(xin))
                ax = tuple(range(xa.dim() - 1))
                xh = (xa - mu) * rstd
                self.bn[(op, "sums")] = ((dya * g).sum(ax), (dya * g * xh).sum(ax))
                self.pgrad[gid] += (dya * xh).sum(ax)
                self.pgrad[bid] += dya.sum(ax)
            sa, sb = self.bn[(op, "sums")]
            m = math.prod(self.ts[xin]["shape"][:-1])
            xh = (x[0] - mu) * rstd
            grads = {xin: rstd * (dy * g - sa / m - xh * sb / m)}
        elif kd == "maxpool":
            grads = {ins[0]: maxpool_bwd(dy, x[0], ia[0], ia[1], ia[2])}
        elif kd in ("relu", "tanh", "add"):  # these save their output (or nothing)
            if kd == "add":
                grads = {}
                for t in ins:
                    grads[t] = grads[t] + dy if t in grads else dy
            else:
                y = self.c(self.store[(out, k)])
                grads = {ins[0]: dy * (y > 0) if kd == "relu" else dy * (1.0 - y * y)}
        else:
            leaves = {}
            xs = []
            for t, v in zip(ins, x):
                if v.dtype.is_floating_point and t in self.needs_grad:
                    v = v.detach().requires_grad_(True)
                    leaves[t] = v
                xs.append(v)
            with torch.enable_grad():
                y = evaluate(xs)
                order = list(leaves)
                gs = torch.autograd.grad(y, [leaves[t] for t in order], grad_outputs=dy, allow_unused=True)
            grads = {t: g for t, g in zip(order, gs) if g is not None}
        for i, t in enumerate(ins):
            g = grads.get(t)
            if g is None:
                continue
            if t in self.pgrad:
                if t in sliced:
                    self.pgrad[t][blk] += g.to(self.pgrad[t].dtype)
                else:
                    self.pgrad[t] += g.to(self.pgrad[t].dtype)
            elif t not in self.needs_grad or self.ts[t]["kind"] != "act":
                continue
            elif st and i == 0:
                self._scatter(t, b0, nb, rect[0], rect[1], rect[2], rect[3], g)
            elif (cm or am) and (self.chan(t) or self.band(t)) and kd not in ("linear", "conv2d"):
                v = self.store[(self.n + t, k)]
                v.copy_((self.c(v) + g).to(v.dtype))
            else:  # a linear / conv reading every block (or the unsplit tensor): dX of its samples
                for blk_, sl in self._pieces(t, b0, b0 + nb, grad=True):
                    blk_.copy_((self.c(blk_) + g[sl]).to(blk_.dtype))

    def _acc(self, t, s0, s1, g):
        if t in self.pgrad:
            self.pgrad[t] += g.to(self.pgrad[t].dtype)
        elif t in self.needs_grad and self.ts[t]["kind"] == "act":
            v = self.view(t, s0, s1, grad=True)
            v.copy_((self.c(v) + g).to(v.dtype))

    def _backward(self, op, k, step):
        o = self.ops[op]
        kd, ia, fa = o["kind"], o["iattrs"], o["fattrs"]
        P = self.P_op(op)
        s0, s1 = k * self.B // P, (k + 1) * self.B // P
        row0, elem0 = self._offsets(op, s0)
        ins, outs = o["inputs"], o["outputs"]
        out = outs[0]
        dy = None if kd == "xent" else self.c(self.view(out, s0, s1, grad=True))

        def val(t):
            v = self.pval[t] if t in self.pval else (self.view(t, s0, s1) if self.sample[t] else self.store[(t, 0)])
            return self.c(v) if v.dtype.is_floating_point else v

        if kd == "relu":
            self._acc(ins[0], s0, s1, dy * (val(out) > 0))
        elif kd == "tanh":
            y = val(out)
            self._acc(ins[0], s0, s1, dy * (1.0 - y * y))
        elif kd == "softmax":
            y = val(out)
            self._acc(ins[0], s0, s1, y * (dy - (dy * y).sum(-1, keepdim=True)))
        elif kd == "add":
            for t in ins:
                self._acc(t, s0, s1, dy)
        elif kd == "dropout":
            g = dy if fa[0] == 0.0 else torch.where(
                dropout_keep(tuple(dy.shape), elem0, fa[0], ia[0], step, dy.device), dy / (1.0 - fa[0]),
                torch.zeros_like(dy))
            self._acc(ins[0], s0, s1, g)
        elif kd == "cls":
            dx = torch.zeros((dy.shape[0] * ia[0], dy.shape[1]), dtype=dy.dtype, device=dy.device)
            dx[::ia[0]] = dy
            self._acc(ins[0], s0, s1, dx)
        elif kd == "avgpool":
            sh = self.ts[ins[0]]["shape"]
            self._acc(ins[0], s0, s1, (dy[:, None, None, :] / (sh[1] * sh[2])).expand(
                (dy.shape[0],) + tuple(sh[1:])))
        elif kd == "flatten":
            sh = self.ts[ins[0]]["shape"]
            self._acc(ins[0], s0, s1, dy.reshape((dy.shape[0],) + tuple(sh[1:])))
        elif kd == "maxpool":
            self._acc(ins[0], s0, s1, maxpool_bwd(dy, val(ins[0]), ia[0], ia[1], ia[2]))
        elif kd == "embed":
            ids, tt = val(ins[0]).long(), val(ins[1]).long()
            pos = torch.arange(row0, row0 + ids.shape[0], device=dy.device) % ia[0]
            self.pgrad[ins[2]].index_add_(0, ids, dy.to(self.pgrad[ins[2]].dtype))
            self.pgrad[ins[3]].index_add_(0, pos, dy.to(self.pgrad[ins[3]].dtype))
            self.pgrad[ins[4]].index_add_(0, tt, dy.to(self.pgrad[ins[4]].dtype))
        elif kd == "batchnorm":
            xin, gid, bid = ins
            mu, var = self.bn[op]
            rstd = 1.0 / torch.sqrt(var + fa[0])
            g = self.pval[gid]
            if k == 0:  # full-batch sums over every piece of dY and X (R13)
                dya, xa = self.c(self.whole(out, grad=True)), self.c(self.whole(xin))
                ax = tuple(range(xa.dim() - 1))
                xh = (xa - mu) * rstd
                self.bn[(op, "sums")] = ((dya * g).sum(ax), (dya * g * xh).sum(ax))
                self.pgrad[gid] += (dya * xh).sum(ax)
                self.pgrad[bid] += dya.sum(ax)
            sa, sb = self.bn[(op, "sums")]
            m = math.prod(self.ts[xin]["shape"][:-1])
            xh = (val(xin) - mu) * rstd
            self._acc(xin, s0, s1, rstd * (dy * g - sa / m - xh * sb / m))
        else:  # autograd on the re-executed micro-op (ops whose backward reads their inputs)
            leaves = {}
            x = []
            for t in ins:
                v = val(t)
                if v.dtype.is_floating_point and t in self.needs_grad:
                    v = v.detach().requires_grad_(True)
                    leaves[t] = v
                x.append(v)
            with torch.enable_grad():
                if kd == "attention":
                    keep = unpack_mask_words(self.view(outs[2], s0, s1), ia[1]) if fa[1] > 0.0 else None
                    y = attention(x[0], x[1], x[2], ia[0], ia[1], fa[0], fa[1], ia[2], 0, step, keep=keep)[0]
                elif kd == "xent":
                    y = xent(x[0], x[1], self.B)
                else:
                    y = self._fwd_op(kd, x, ia, fa, row0, elem0, step)
                order = list(leaves)
                gs = torch.autograd.grad(y, [leaves[t] for t in order], grad_outputs=None if kd == "xent" else dy,
                                         allow_unused=True)
            for t, g in zip(order, gs):
                if g is not None:
                    self._acc(t, s0, s1, g)
