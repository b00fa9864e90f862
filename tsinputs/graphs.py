"""Workload dataflow graphs (DFGs) — plain data, no arithmetic of the method.

The DFG is the *input* of TSPLIT (§II: "the computation of DNNs is
typically expressed as a dataflow graph (DFG) ... nodes are operations, and the
edges are tensors"; Alg. 1 "Data: G: Computation Graph", L62-75).  This module
only lists tensors (name, dtype, shape, kind) and operations (kind, inputs,
outputs, attributes) for the networks named in BASELINE.json's configs.  Both
the fp64 oracle (`oracle/`) and the product binding consume these lists; neither
side's computation lives here.

Tensor kinds: "param" (model weights, static region), "input" (sample data),
"label", "act" (activations produced by an op).  Every non-param tensor except
the scalar loss has a leading *sample* dimension of `samples` (batch) units —
the dimension TSPLIT splits along ("split along the dim of sample").

Operation kinds and attributes (semantics in DESIGN.md §3):
  linear     in (X[R,K], W[N,K], b[N])      out Y[R,N] = X W^T + b
  relu/gelu/tanh  in (X)                    out elementwise
  layernorm  in (X[R,H], gamma[H], beta[H]) out;  f: eps
  add        in (A, B)                      out A + B
  dropout    in (X)                         out; f: p, i: seed (Philox counter)
  softmax    in (X[..., L])                 out row softmax over the last dim
  attn_qk    in (Q[T,h], K[T,h])            out S[b,a,s,s] = alpha Q_h K_h^T; i: heads, seq; f: alpha
  attn_pv    in (P[b,a,s,s], V[T,h])        out C[T,h] (heads re-merged); i: heads, seq
  embed      in (ids[T], tt[T], Wword[V,h], Wpos[S,h], Wtype[2,h])  out [T,h]; i: seq
  cls        in (X[T,h])                    out [b,h] = rows b*seq; i: seq
  xent       in (logits[b,C], labels[b])    out loss[1] = mean_b CE (global batch)
"""

from __future__ import annotations

import math

DTYPE_BYTES = {"f32": 4, "bf16": 2, "i32": 4}


class GraphBuilder:
    def __init__(self, name: str, dtype: str, samples: int):
        self.name = name
        self.dtype = dtype
        self.samples = samples
        self.tensors: list[dict] = []
        self.ops: list[dict] = []

    def tensor(self, name, shape, kind, dtype=None):
        t = {
            "id": len(self.tensors),
            "name": name,
            "dtype": dtype or self.dtype,
            "shape": tuple(int(s) for s in shape),
            "kind": kind,
        }
        self.tensors.append(t)
        return t["id"]

    def param(self, name, shape):
        return self.tensor(name, shape, "param")

    def op(self, kind, name, inputs, out_shape, out_name=None, iattrs=(), fattrs=(), out_dtype=None):
        out = self.tensor(out_name or name, out_shape, "act", dtype=out_dtype)
        self.ops.append({
            "id": len(self.ops),
            "kind": kind,
            "name": name,
            "inputs": list(inputs),
            "outputs": [out],
            "iattrs": [int(v) for v in iattrs],
            "fattrs": [float(v) for v in fattrs],
        })
        return out

    def op_multi(self, kind, name, inputs, outs, iattrs=(), fattrs=()):
        """An op with several outputs: outs = [(name, shape, dtype or None)]."""
        ids = [self.tensor(n, sh, "act", dtype=dt) for n, sh, dt in outs]
        self.ops.append({
            "id": len(self.ops),
            "kind": kind,
            "name": name,
            "inputs": list(inputs),
            "outputs": ids,
            "iattrs": [int(v) for v in iattrs],
            "fattrs": [float(v) for v in fattrs],
        })
        return ids

    def done(self) -> dict:
        return {
            "name": self.name,
            "dtype": self.dtype,
            "samples": self.samples,
            "tensors": self.tensors,
            "ops": self.ops,
        }


def mlp(batch=8, hidden=256, depth=3, in_dim=256, classes=10, dtype="f32") -> dict:
    """Config 1 (BASELINE.json configs[0]): 3-layer MLP 256->256->256->10, ReLU.

    5 forward ops + loss.
    """
    g = GraphBuilder(f"mlp{depth}_h{hidden}_b{batch}", dtype, batch)
    x = g.tensor("x", (batch, in_dim), "input")
    y = g.tensor("labels", (batch,), "label", dtype="i32")
    h = x
    dims = [in_dim] + [hidden] * (depth - 1) + [classes]
    for li in range(depth):
        w = g.param(f"fc{li}.w", (dims[li + 1], dims[li]))
        b = g.param(f"fc{li}.b", (dims[li + 1],))
        h = g.op("linear", f"fc{li}", [h, w, b], (batch, dims[li + 1]))
        if li < depth - 1:
            h = g.op("relu", f"relu{li}", [h], (batch, dims[li + 1]))
    g.op("xent", "loss", [h, y], (1,), out_dtype="f32")
    return g.done()


def bert(layers=24, hidden=1024, heads=16, seq=512, batch=32, vocab=30522, ffn=None,
         classes=2, dtype="bf16", attn_dropout=0.1, emb_dropout=0.1, seed=1234,
         fused_attention=False) -> dict:
    """Canonical unfused BERT encoder + pooler/classifier head (MRPC-like).

    Per layer it emits exactly the tensors SURVEY.md §4 T2 reconciles with
    PAPER.md Table II (L85-112): 3 x [b,a,s,s] (scores, softmax, attention
    dropout), 2 x [T,4h] (FFN1, GELU), 10 x [T,h] (Q, K, V, context, proj, res1,
    LN1, FFN2, res2, LN2), weights 2 x [h,4h] and 4 x [h,h].

    fused_attention=True replaces scores/probs/attn_drop/ctx by
    one "attention" op: in (Q, K, V), out (ctx [T,h], lse [b,a,s] f32, dropout keep
    bits [b,a,s,s/32] i32); iattrs {heads, seq, dropout seed}, fattrs {alpha, p}; the
    same function (same seeds).
    """
    ffn = ffn or 4 * hidden
    assert hidden % heads == 0
    dh = hidden // heads
    T = batch * seq
    g = GraphBuilder(f"bert_L{layers}_h{hidden}_a{heads}_s{seq}_b{batch}" + ("_fa" if fused_attention else ""),
                     dtype, batch)
    ids = g.tensor("input_ids", (T,), "input", dtype="i32")
    tts = g.tensor("token_type_ids", (T,), "input", dtype="i32")
    labels = g.tensor("labels", (batch,), "label", dtype="i32")
    wword = g.param("emb.word", (vocab, hidden))
    wpos = g.param("emb.pos", (seq, hidden))
    wtype = g.param("emb.type", (2, hidden))
    e = g.op("embed", "emb", [ids, tts, wword, wpos, wtype], (T, hidden), iattrs=[seq])
    lg = g.param("emb.ln.g", (hidden,))
    lb = g.param("emb.ln.b", (hidden,))
    e = g.op("layernorm", "emb.ln", [e, lg, lb], (T, hidden), fattrs=[1e-12])
    x = g.op("dropout", "emb.drop", [e], (T, hidden), fattrs=[emb_dropout], iattrs=[seed])
    alpha = 1.0 / math.sqrt(dh)
    for l in range(layers):
        p = f"l{l}."

        def lin(name, inp, n_out, n_in):
            w = g.param(p + name + ".w", (n_out, n_in))
            b = g.param(p + name + ".b", (n_out,))
            return g.op("linear", p + name, [inp, w, b], (T, n_out))

        q = lin("q", x, hidden, hidden)
        k = lin("k", x, hidden, hidden)
        v = lin("v", x, hidden, hidden)
        if fused_attention:
            c, _, _ = g.op_multi("attention", p + "attn", [q, k, v],
                                 [(p + "ctx", (T, hidden), None), (p + "lse", (batch, heads, seq), "f32"),
                                  (p + "dmask", (batch, heads, seq, seq // 32), "i32")],
                                 iattrs=[heads, seq, seed + 1 + l], fattrs=[alpha, attn_dropout])
        else:
            s = g.op("attn_qk", p + "scores", [q, k], (batch, heads, seq, seq), iattrs=[heads, seq],
                     fattrs=[alpha])
            pr = g.op("softmax", p + "probs", [s], (batch, heads, seq, seq))
            pd = g.op("dropout", p + "attn_drop", [pr], (batch, heads, seq, seq), fattrs=[attn_dropout],
                      iattrs=[seed + 1 + l])
            c = g.op("attn_pv", p + "ctx", [pd, v], (T, hidden), iattrs=[heads, seq])
        o = lin("proj", c, hidden, hidden)
        r1 = g.op("add", p + "res1", [o, x], (T, hidden))
        g1 = g.param(p + "ln1.g", (hidden,))
        b1 = g.param(p + "ln1.b", (hidden,))
        n1 = g.op("layernorm", p + "ln1", [r1, g1, b1], (T, hidden), fattrs=[1e-12])
        f1 = lin("ffn1", n1, ffn, hidden)
        ge = g.op("gelu", p + "gelu", [f1], (T, ffn))
        f2 = lin("ffn2", ge, hidden, ffn)
        r2 = g.op("add", p + "res2", [f2, n1], (T, hidden))
        g2 = g.param(p + "ln2.g", (hidden,))
        b2 = g.param(p + "ln2.b", (hidden,))
        x = g.op("layernorm", p + "ln2", [r2, g2, b2], (T, hidden), fattrs=[1e-12])
    cls = g.op("cls", "pool.cls", [x], (batch, hidden), iattrs=[seq])
    pw = g.param("pool.w", (hidden, hidden))
    pb = g.param("pool.b", (hidden,))
    pl = g.op("linear", "pool.fc", [cls, pw, pb], (batch, hidden))
    pt = g.op("tanh", "pool.tanh", [pl], (batch, hidden))
    cw = g.param("cls.w", (classes, hidden))
    cb = g.param("cls.b", (classes,))
    lo = g.op("linear", "cls.fc", [pt, cw, cb], (batch, classes))
    g.op("xent", "loss", [lo, labels], (1,), out_dtype="f32")
    return g.done()


def transformer(enc_layers=6, dec_layers=6, hidden=512, heads=8, ffn=2048, seq=128, batch=64, vocab=32000,
                dtype="bf16", dropout=0.1, seed=4321) -> dict:
    """Encoder-decoder Transformer shaped like the paper's IWSLT2016 workload (P:L306:
    "the IWSLT2016 dataset for Transformer"), source and target of `seq`
    tokens, post-LN layers as in bert().  Encoder layer: self-attention (fused op, no mask)
    + add&LN + FFN + add&LN.  Decoder layer: causal self-attention (unfused: attn_qk ->
    softmax(causal) -> dropout -> attn_pv), add&LN, cross-attention (q from the decoder,
    k / v from the encoder output; equal lengths, so the same attention op) + add&LN,
    FFN + add&LN.  Head: linear to the target vocabulary and the token-level cross
    entropy (labels [T]): the loss is the per-sentence sum of token losses, averaged over
    the batch (R14: mean over the global batch of samples)."""
    assert hidden % heads == 0
    dh = hidden // heads
    T = batch * seq
    g = GraphBuilder(f"transformer_E{enc_layers}D{dec_layers}_h{hidden}_a{heads}_s{seq}_b{batch}", dtype, batch)
    src = g.tensor("src_ids", (T,), "input", dtype="i32")
    tgt = g.tensor("tgt_ids", (T,), "input", dtype="i32")
    seg = g.tensor("token_type_ids", (T,), "input", dtype="i32")
    labels = g.tensor("tgt_labels", (T,), "label", dtype="i32")
    alpha = 1.0 / math.sqrt(dh)
    sd = [seed]

    def nseed():
        sd[0] += 1
        return sd[0]

    def embed(name, ids):
        w = g.param(name + ".word", (vocab, hidden))
        p = g.param(name + ".pos", (seq, hidden))
        ty = g.param(name + ".type", (2, hidden))
        e = g.op("embed", name, [ids, seg, w, p, ty], (T, hidden), iattrs=[seq])
        e = ln(name + ".ln", e)
        return g.op("dropout", name + ".drop", [e], (T, hidden), fattrs=[dropout], iattrs=[nseed()])

    def lin(name, inp, n_out, n_in):
        w = g.param(name + ".w", (n_out, n_in))
        b = g.param(name + ".b", (n_out,))
        return g.op("linear", name, [inp, w, b], (T, n_out))

    def ln(name, x):
        gm = g.param(name + ".g", (hidden,))
        bt = g.param(name + ".b", (hidden,))
        return g.op("layernorm", name, [x, gm, bt], (T, hidden), fattrs=[1e-12])

    def fused_attn(p, xq, xkv):
        q = lin(p + "q", xq, hidden, hidden)
        k = lin(p + "k", xkv, hidden, hidden)
        v = lin(p + "v", xkv, hidden, hidden)
        c, _, _ = g.op_multi("attention", p + "attn", [q, k, v],
                             [(p + "ctx", (T, hidden), None), (p + "lse", (batch, heads, seq), "f32"),
                              (p + "dmask", (batch, heads, seq, seq // 32), "i32")],
                             iattrs=[heads, seq, nseed()], fattrs=[alpha, dropout])
        return lin(p + "proj", c, hidden, hidden)

    def causal_attn(p, x):
        q = lin(p + "q", x, hidden, hidden)
        k = lin(p + "k", x, hidden, hidden)
        v = lin(p + "v", x, hidden, hidden)
        s = g.op("attn_qk", p + "scores", [q, k], (batch, heads, seq, seq), iattrs=[heads, seq], fattrs=[alpha])
        pr = g.op("softmax", p + "probs", [s], (batch, heads, seq, seq), iattrs=[1])
        pd = g.op("dropout", p + "attn_drop", [pr], (batch, heads, seq, seq), fattrs=[dropout], iattrs=[nseed()])
        c = g.op("attn_pv", p + "ctx", [pd, v], (T, hidden), iattrs=[heads, seq])
        return lin(p + "proj", c, hidden, hidden)

    def mlp_block(p, x):
        f1 = lin(p + "ffn1", x, ffn, hidden)
        ge = g.op("gelu", p + "gelu", [f1], (T, ffn))
        return lin(p + "ffn2", ge, hidden, ffn)

    x = embed("src", src)
    for l in range(enc_layers):
        p = f"e{l}."
        x = ln(p + "ln1", g.op("add", p + "res1", [fused_attn(p, x, x), x], (T, hidden)))
        x = ln(p + "ln2", g.op("add", p + "res2", [mlp_block(p, x), x], (T, hidden)))
    enc = x
    y = embed("tgt", tgt)
    for l in range(dec_layers):
        p = f"d{l}."
        y = ln(p + "ln1", g.op("add", p + "res1", [causal_attn(p + "self.", y), y], (T, hidden)))
        y = ln(p + "ln2", g.op("add", p + "res2", [fused_attn(p + "cross.", y, enc), y], (T, hidden)))
        y = ln(p + "ln3", g.op("add", p + "res3", [mlp_block(p, y), y], (T, hidden)))
    logits = lin("out", y, vocab, hidden)
    g.op("xent", "loss", [logits, labels], (1,), out_dtype="f32")
    return g.done()


def tensor_bytes(t: dict) -> int:
    n = 1
    for s in t["shape"]:
        n *= s
    return n * DTYPE_BYTES[t["dtype"]]


def config_graph(name: str, **over) -> dict:
    """Graphs for BASELINE.json configs by short name."""
    if name == "mlp":
        return mlp(**over)
    if name == "bert_large":
        kw = dict(layers=24, hidden=1024, heads=16, seq=512, batch=32)
        kw.update(over)
        return bert(**kw)
    if name == "bert_tiny":
        kw = dict(layers=2, hidden=128, heads=2, seq=64, batch=4, vocab=512)
        kw.update(over)
        return bert(**kw)
    if name == "bert_small":  # the bf16 parity size (DESIGN.md D-TOL): hidden 256, 4 heads of 64
        kw = dict(layers=2, hidden=256, heads=4, seq=128, batch=8, vocab=512)
        kw.update(over)
        return bert(**kw)
    if name == "vgg16":
        return vgg16(**over)
    if name == "vgg_tiny":
        kw = dict(batch=4, img=32, width=0.125, fc=64, classes=10,
                  cfg=[64, "M", 128, "M", 256, 256, "M"])
        kw.update(over)
        return vgg16(**kw)
    if name == "vgg_small":  # bf16 precision study size (DESIGN.md D-TOL)
        kw = dict(batch=16, img=32, width=0.25, fc=128, classes=10,
                  cfg=[64, "M", 128, "M", 256, 256, "M"])
        kw.update(over)
        return vgg16(**kw)
    if name == "resnet50":
        return resnet50(**over)
    if name == "resnet_tiny":
        kw = dict(batch=4, img=32, width=0.125, blocks=(1, 1), classes=10)
        kw.update(over)
        return resnet50(**kw)
    if name == "resnet_small":
        kw = dict(batch=16, img=32, width=0.25, blocks=(1, 1), classes=10)
        kw.update(over)
        return resnet50(**kw)
    if name == "transformer_iwslt":  # f4 workload, IWSLT-shaped
        return transformer(**over)
    if name == "transformer_tiny":
        kw = dict(enc_layers=1, dec_layers=1, hidden=128, heads=2, ffn=256, seq=64, batch=4, vocab=512)
        kw.update(over)
        return transformer(**kw)
    if name == "transformer_small":  # the bf16 parity size
        kw = dict(enc_layers=1, dec_layers=2, hidden=256, heads=4, ffn=1024, seq=128, batch=8, vocab=1024)
        kw.update(over)
        return transformer(**kw)
    if name == "bert_scaled":
        kw = dict(layers=24, hidden=2560, heads=40, seq=512, batch=64)
        kw.update(over)
        return bert(**kw)
    raise KeyError(name)


def _conv_out(h, k, stride, pad):
    return (h + 2 * pad - k) // stride + 1


def vgg16(batch=64, img=224, classes=1000, width=1.0, fc=4096, dtype="bf16", cfg=None) -> dict:
    """Config 2 (BASELINE configs[1]): VGG-16 (13 conv3x3 + ReLU, 5 maxpool 2x2/2,
    3 FC), NHWC activations, KRSC weights; `width` scales the channels (Table V's
    parameter scale)."""
    cfg = cfg or [64, 64, "M", 128, 128, "M", 256, 256, 256, "M", 512, 512, 512, "M", 512, 512, 512, "M"]
    g = GraphBuilder(f"vgg16_b{batch}_i{img}_w{width}", dtype, batch)
    x = g.tensor("image", (batch, img, img, 3), "input")
    y = g.tensor("labels", (batch,), "label", dtype="i32")
    h, c, li = img, 3, 0
    for v in cfg:
        if v == "M":
            h = _conv_out(h, 2, 2, 0)
            x = g.op("maxpool", f"pool{li}", [x], (batch, h, h, c), iattrs=[2, 2, 0])
            continue
        k = max(8, int(v * width))
        w = g.param(f"conv{li}.w", (k, 3, 3, c))
        b = g.param(f"conv{li}.b", (k,))
        x = g.op("conv2d", f"conv{li}", [x, w, b], (batch, h, h, k), iattrs=[1, 1])
        x = g.op("relu", f"relu{li}", [x], (batch, h, h, k))
        c = k
        li += 1
    x = g.op("flatten", "flatten", [x], (batch, h * h * c))
    dims = [h * h * c, fc, fc, classes]
    for i in range(3):
        w = g.param(f"fc{i}.w", (dims[i + 1], dims[i]))
        b = g.param(f"fc{i}.b", (dims[i + 1],))
        x = g.op("linear", f"fc{i}", [x, w, b], (batch, dims[i + 1]))
        if i < 2:
            x = g.op("relu", f"fcrelu{i}", [x], (batch, dims[i + 1]))
    g.op("xent", "loss", [x, y], (1,), out_dtype="f32")
    return g.done()


def resnet50(batch=256, img=224, classes=1000, width=1.0, blocks=(3, 4, 6, 3), dtype="bf16") -> dict:
    """Config 3 (BASELINE configs[2]): ResNet-50 v1.5 (stride on the 3x3 conv of each
    stage's first bottleneck), conv without bias + train-mode BN, NHWC."""
    g = GraphBuilder(f"resnet50_b{batch}_i{img}_w{width}", dtype, batch)
    x = g.tensor("image", (batch, img, img, 3), "input")
    y = g.tensor("labels", (batch,), "label", dtype="i32")
    cnt = [0]

    def conv_bn(name, x, cin, cout, k, stride, h, relu=True):
        pad = k // 2
        ho = _conv_out(h, k, stride, pad)
        w = g.param(name + ".w", (cout, k, k, cin))
        x = g.op("conv2d", name, [x, w], (batch, ho, ho, cout), iattrs=[stride, pad])
        gm = g.param(name + ".bn.g", (cout,))
        bt = g.param(name + ".bn.b", (cout,))
        x = g.op("batchnorm", name + ".bn", [x, gm, bt], (batch, ho, ho, cout), fattrs=[1e-5])
        if relu:
            x = g.op("relu", name + ".relu", [x], (batch, ho, ho, cout))
        return x, ho

    c0 = max(8, int(64 * width))
    x, h = conv_bn("stem", x, 3, c0, 7, 2, img)
    h2 = _conv_out(h, 3, 2, 1)
    x = g.op("maxpool", "stem.pool", [x], (batch, h2, h2, c0), iattrs=[3, 2, 1])
    h, cin = h2, c0
    for si, nb in enumerate(blocks):
        mid = max(8, int(64 * width * 2 ** si))
        cout = 4 * mid
        for bi in range(nb):
            stride = 2 if (bi == 0 and si > 0) else 1
            p = f"s{si}b{bi}"
            a, ha = conv_bn(p + ".c1", x, cin, mid, 1, 1, h)
            a, hb = conv_bn(p + ".c2", a, mid, mid, 3, stride, ha)
            a, hc = conv_bn(p + ".c3", a, mid, cout, 1, 1, hb, relu=False)
            if bi == 0:
                sc, _ = conv_bn(p + ".down", x, cin, cout, 1, stride, h, relu=False)
            else:
                sc = x
            s = g.op("add", p + ".add", [a, sc], (batch, hc, hc, cout))
            x = g.op("relu", p + ".relu", [s], (batch, hc, hc, cout))
            h, cin = hc, cout
    x = g.op("avgpool", "avgpool", [x], (batch, cin))
    w = g.param("fc.w", (classes, cin))
    b = g.param("fc.b", (classes,))
    x = g.op("linear", "fc", [x, w, b], (batch, classes))
    g.op("xent", "loss", [x, y], (1,), out_dtype="f32")
    return g.done()
