"""ORACLE — test infrastructure only.

Unsplit fp64 training step of a DFG (§II: feed-forward pass, loss
L, back-propagation "to obtain the gradients dL/dw of each model parameter").
This is the plain definition every TSPLIT plan must reproduce (T1).
Ops run in definition order (the tsinputs builders emit a topological order);
the backward pass visits ops in reverse and sums gradient contributions.
"""

from __future__ import annotations

import numpy as np

from . import ops

F = np.float64


def _attrs(op):
    return op["iattrs"], op["fattrs"]


def forward_op(graph, op, val, row0=0, elem0=0, step=0):
    """Evaluate one op on `val` (tensor id -> fp64/int array) for a block of samples
    starting at global sample-row `row0` / element `elem0` of the output."""
    k = op["kind"]
    ia, fa = _attrs(op)
    x = [val[i] for i in op["inputs"]]
    if k == "linear":
        return ops.linear_fwd(x[0], x[1], x[2])
    if k == "relu":
        return ops.relu_fwd(x[0])
    if k == "gelu":
        return ops.gelu_fwd(x[0])
    if k == "tanh":
        return ops.tanh_fwd(x[0])
    if k == "layernorm":
        return ops.layernorm_fwd(x[0], x[1], x[2], fa[0])
    if k == "add":
        return ops.add_fwd(x[0], x[1])
    if k == "dropout":
        return ops.dropout_fwd(x[0], fa[0], ia[0], elem0, step)
    if k == "softmax":
        return ops.softmax_fwd(x[0], causal=bool(ia and ia[0]))
    if k == "attn_qk":
        return ops.attn_qk_fwd(x[0], x[1], ia[0], ia[1], fa[0])
    if k == "attn_pv":
        return ops.attn_pv_fwd(x[0], x[1], ia[0], ia[1])
    if k == "attention":  # outputs (C, lse, keep-mask words); dropout offset from the first sample
        b0 = row0 // ia[1]
        return ops.attention_fwd(x[0], x[1], x[2], ia[0], ia[1], fa[0], fa[1], ia[2],
                                 b0 * ia[0] * ia[1] * ia[1], step)
    if k == "embed":
        return ops.embed_fwd(x[0], x[1], x[2], x[3], x[4], ia[0], row0)
    if k == "cls":
        return ops.cls_fwd(x[0], ia[0])
    if k == "xent":
        return np.array([ops.xent_fwd(x[0], x[1], graph["samples"])])
    if k == "conv2d":
        return ops.conv2d_fwd(x[0], x[1], x[2] if len(x) > 2 else None, ia[0], ia[1])
    if k == "batchnorm":
        return ops.batchnorm_fwd(x[0], x[1], x[2], fa[0])
    if k == "maxpool":
        return ops.maxpool_fwd(x[0], ia[0], ia[1], ia[2])
    if k == "avgpool":
        return ops.avgpool_fwd(x[0])
    if k == "flatten":
        return x[0].reshape(x[0].shape[0], -1).copy()
    raise ValueError(k)


def backward_op(graph, op, val, dy, row0=0, elem0=0, step=0):
    """Returns {tensor id: gradient contribution} for the op's inputs.

    `dy` is the gradient of the op's output (None for xent, whose output is L)."""
    k = op["kind"]
    ia, fa = _attrs(op)
    ins = op["inputs"]
    x = [val.get(i) for i in ins]
    out = {}
    if k == "linear":
        dx, dw, db = ops.linear_bwd(dy, x[0], x[1])
        out = {ins[0]: dx, ins[1]: dw, ins[2]: db}
    elif k == "relu":
        out = {ins[0]: ops.relu_bwd(dy, val[op["outputs"][0]])}
    elif k == "gelu":
        out = {ins[0]: ops.gelu_bwd(dy, x[0])}
    elif k == "tanh":
        out = {ins[0]: ops.tanh_bwd(dy, val[op["outputs"][0]])}
    elif k == "layernorm":
        dx, dg, db = ops.layernorm_bwd(dy, x[0], x[1], fa[0])
        out = {ins[0]: dx, ins[1]: dg, ins[2]: db}
    elif k == "add":
        out = {ins[0]: dy, ins[1]: dy}
    elif k == "dropout":
        out = {ins[0]: ops.dropout_bwd(dy, fa[0], ia[0], elem0, step)}
    elif k == "softmax":
        out = {ins[0]: ops.softmax_bwd(dy, val[op["outputs"][0]])}
    elif k == "attn_qk":
        dq, dk = ops.attn_qk_bwd(dy, x[0], x[1], ia[0], ia[1], fa[0])
        out = {ins[0]: dq, ins[1]: dk}
    elif k == "attn_pv":
        dp, dv = ops.attn_pv_bwd(dy, x[0], x[1], ia[0], ia[1])
        out = {ins[0]: dp, ins[1]: dv}
    elif k == "attention":
        b0 = row0 // ia[1]
        dq, dk, dv = ops.attention_bwd(dy, x[0], x[1], x[2], ia[0], ia[1], fa[0], fa[1], ia[2],
                                       b0 * ia[0] * ia[1] * ia[1], step)
        out = {ins[0]: dq, ins[1]: dk, ins[2]: dv}
    elif k == "embed":
        shapes = [graph["tensors"][i]["shape"] for i in ins[2:5]]
        dw, dp, dt = ops.embed_bwd(dy, x[0], x[1], ia[0], row0, shapes)
        out = {ins[2]: dw, ins[3]: dp, ins[4]: dt}
    elif k == "cls":
        rows = dy.shape[0] * ia[0]
        out = {ins[0]: ops.cls_bwd(dy, ia[0], rows)}
    elif k == "xent":
        out = {ins[0]: ops.xent_bwd(x[0], x[1], graph["samples"])}
    elif k == "conv2d":
        dx, dw, db = ops.conv2d_bwd(dy, x[0], x[1], ia[0], ia[1])
        out = {ins[0]: dx, ins[1]: dw}
        if len(ins) > 2:
            out[ins[2]] = db
    elif k == "batchnorm":
        dx, dg, db = ops.batchnorm_bwd(dy, x[0], x[1], fa[0])
        out = {ins[0]: dx, ins[1]: dg, ins[2]: db}
    elif k == "maxpool":
        out = {ins[0]: ops.maxpool_bwd(dy, x[0], ia[0], ia[1], ia[2])}
    elif k == "avgpool":
        shape = (dy.shape[0],) + tuple(graph["tensors"][ins[0]]["shape"][1:])
        out = {ins[0]: ops.avgpool_bwd(dy, shape)}
    elif k == "flatten":
        shape = (dy.shape[0],) + tuple(graph["tensors"][ins[0]]["shape"][1:])
        out = {ins[0]: dy.reshape(shape).copy()}
    else:
        raise ValueError(k)
    return out


# Auxiliary outputs: statistics an op saves for its own backward, never read by another
# op and never differentiated (the fused attention's row log-sum-exp).
AUX_OUTPUTS = {"attention": (1, 2)}


def grad_outputs(op):
    """The outputs of `op` that carry a gradient."""
    aux = AUX_OUTPUTS.get(op["kind"], ())
    return [t for i, t in enumerate(op["outputs"]) if i not in aux]


def needs_grad(graph):
    """Tensor ids that carry a gradient: params, and activations downstream of one."""
    ng = {t["id"] for t in graph["tensors"] if t["kind"] == "param"}
    for op in graph["ops"]:
        if any(i in ng for i in op["inputs"]):
            ng.update(grad_outputs(op))
    return ng


def initial_values(graph, params, inputs):
    val = {}
    for t in graph["tensors"]:
        if t["kind"] == "param":
            val[t["id"]] = np.asarray(params[t["name"]], F)
        elif t["kind"] in ("input", "label"):
            a = np.asarray(inputs[t["name"]])
            val[t["id"]] = a.astype(np.int64) if t["dtype"] == "i32" else a.astype(F)
    return val


def train_step(graph, params, inputs, step=0, storage=None):
    """Unsplit fp64 forward + backward.  Returns (loss, {param name: grad}).

    storage="bf16": every stored activation and activation gradient is rounded to
    bf16 (ops.round_bf16) where it is written — after each forward op and after
    each gradient contribution is added — while the arithmetic inside an op stays
    fp64.  That is the precision a bf16-storage / fp32-compute implementation
    keeps, so its gradients are compared against this reading
    (DESIGN.md D-TOL); parameter gradients are never rounded (fp32 masters)."""
    rnd = ops.round_bf16 if storage == "bf16" else (lambda a: a)
    val = initial_values(graph, params, inputs)
    loss_id = next(op["outputs"][0] for op in graph["ops"] if op["kind"] == "xent")
    ts = graph["tensors"]
    for op in graph["ops"]:
        y = forward_op(graph, op, val, step=step)
        ys = y if isinstance(y, tuple) else (y,)
        for t, yt in zip(op["outputs"], ys):
            val[t] = rnd(yt) if ts[t]["dtype"] == "bf16" else yt
    ng = needs_grad(graph)
    is_act = {t["id"] for t in graph["tensors"] if t["kind"] == "act"}
    grad = {}
    for op in reversed(graph["ops"]):
        o = op["outputs"][0]
        if o != loss_id and o not in grad:
            continue
        contrib = backward_op(graph, op, val, grad.get(o), step=step)
        for tid, g in contrib.items():
            if tid not in ng:
                continue
            grad[tid] = grad[tid] + g if tid in grad else g
            if tid in is_act:
                grad[tid] = rnd(grad[tid])
    pg = {t["name"]: grad.get(t["id"], np.zeros(t["shape"]))
          for t in graph["tensors"] if t["kind"] == "param"}
    return float(val[loss_id][0]), pg, val, grad
