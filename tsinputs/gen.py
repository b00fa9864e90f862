"""Seeded synthetic inputs and parameter initialisations (no method arithmetic).

Recipes (DESIGN.md §5 "Input recipe"):
  * MLP (config 1): x ~ N(0,1) [seed 0]; W, b ~ U(+-1/sqrt(fan_in)) [seed 1 + param index];
    labels uniform in [0, classes) [seed 2].
  * Transformer (f4, IWSLT-shaped): source / target ids and next-token labels uniform in
    [0, vocab) [seeds 3000 / 4000 / 5000 + rank]; parameters as BERT's.
  * BERT: token ids uniform in [0, vocab) [seed 1000 + rank]; token-type ids 0 (one
    segment, P:L16 MRPC-like pairs are not modelled); labels uniform in {0,1};
    weights and embeddings ~ N(0, 0.02); biases ~ N(0, 0.02) (non-zero so that bias
    gradients are exercised); LayerNorm gamma ~ 1 + N(0, 0.05), beta ~ N(0, 0.02).
For bf16 graphs every generated float is snapped to the nearest bf16 value here,
so the fp32 master and its bf16 copy coincide at step 0 and both sides start from
the identical operands (the oracle widens them to fp64).
"""

from __future__ import annotations

import zlib

import numpy as np


def snap_bf16(a: np.ndarray) -> np.ndarray:
    """Round fp32 values to the nearest bf16 (ties to even), returned as fp32."""
    a = np.ascontiguousarray(a, dtype=np.float32)
    u = a.view(np.uint32).astype(np.uint64)
    rounded = ((u + 0x7FFF + ((u >> 16) & 1)) >> 16) << 16
    return rounded.astype(np.uint32).view(np.float32).reshape(a.shape)


def _rng(seed: int, name: str) -> np.random.Generator:
    return np.random.default_rng([seed, zlib.crc32(name.encode())])


def init_params(graph: dict, seed: int = 1) -> dict[str, np.ndarray]:
    """fp32 parameter values keyed by tensor name."""
    out = {}
    is_bert = graph["name"].startswith(("bert", "transformer"))  # same recipe for the Transformer
    is_cnn = graph["name"].startswith(("vgg", "resnet"))
    for t in graph["tensors"]:
        if t["kind"] != "param":
            continue
        name, shape = t["name"], t["shape"]
        r = _rng(seed, name)
        if is_cnn:
            if len(shape) == 4:  # conv KRSC: Kaiming-normal, fan_in = R*S*C
                v = np.sqrt(2.0 / (shape[1] * shape[2] * shape[3])) * r.standard_normal(shape)
            elif len(shape) == 2:
                v = np.sqrt(2.0 / shape[1]) * r.standard_normal(shape)
            elif name.endswith(".bn.g"):
                v = 1.0 + 0.1 * r.standard_normal(shape)
            else:
                v = 0.05 * r.standard_normal(shape)
        elif is_bert:
            if name.endswith(".g"):
                v = 1.0 + 0.05 * r.standard_normal(shape)
            else:
                v = 0.02 * r.standard_normal(shape)
        else:
            fan_in = shape[1] if len(shape) == 2 else None
            if fan_in is None:  # bias: fan_in of the weight of the linear op using it
                op = next(o for o in graph["ops"] if o["kind"] == "linear" and o["inputs"][2] == t["id"])
                fan_in = graph["tensors"][op["inputs"][1]]["shape"][1]
            bound = 1.0 / np.sqrt(fan_in)
            v = r.uniform(-bound, bound, size=shape)
        v = v.astype(np.float32)
        if graph["dtype"] == "bf16":
            v = snap_bf16(v)
        out[name] = v
    return out


def make_inputs(graph: dict, seed: int = 0) -> dict[str, np.ndarray]:
    """Input and label arrays keyed by tensor name (ints as int32, floats as fp32)."""
    out = {}
    is_bert = graph["name"].startswith("bert")
    vocab = None
    for t in graph["tensors"]:
        if t["name"] == "emb.word":
            vocab = t["shape"][0]
    xent = next(o for o in graph["ops"] if o["kind"] == "xent")
    classes = graph["tensors"][xent["inputs"][0]]["shape"][1]
    for t in graph["tensors"]:
        if t["kind"] not in ("input", "label"):
            continue
        name, shape = t["name"], t["shape"]
        if graph["name"].startswith("transformer"):  # token ids / next-token labels uniform in the vocab
            tag = {"src_ids": 3000, "tgt_ids": 4000, "tgt_labels": 5000}.get(name)
            if tag is None:
                out[name] = np.zeros(shape, np.int32)
            else:
                out[name] = np.random.default_rng(tag + seed).integers(0, classes, size=shape).astype(np.int32)
        elif is_bert:
            r = np.random.default_rng(1000 + seed)
            if name == "input_ids":
                out[name] = r.integers(0, vocab, size=shape, dtype=np.int64).astype(np.int32)
            elif name == "token_type_ids":
                out[name] = np.zeros(shape, np.int32)
            else:
                out[name] = np.random.default_rng(2000 + seed).integers(0, classes, size=shape).astype(np.int32)
        else:  # MLP features / CNN images: N(0,1); labels uniform in [0, classes)
            if t["kind"] == "input":
                v = np.random.default_rng(seed).standard_normal(shape).astype(np.float32)
                if graph["dtype"] == "bf16":
                    v = snap_bf16(v)
                out[name] = v
            else:
                out[name] = np.random.default_rng(seed + 2).integers(0, classes, size=shape).astype(np.int32)
    return out
