"""ORACLE — test infrastructure only (see oracle/__init__.py).

Plain fp64 numpy forward and vector-Jacobian products of the operations the
DFGs in tsinputs.graphs use.  TSPLIT itself does not change any operator
(§VI-D: "TSPLIT will not result in changes in existing operator
implementation"; L42: swap/recompute have "no accuracy loss"), so the numeric
oracle is the plain textbook definition of each op, evaluated unsplit.
Silent points of the paper are taken as SURVEY.md §8(c) R15/R16 read them:
erf-GELU, biased LayerNorm variance, attention scale 1/sqrt(d_head) without a
padding mask, Philox-keyed dropout, mean cross-entropy over the *global* batch
(R14).  Every function works on a contiguous block of samples; `row0`/`elem0`
give the global offset of that block so that position embeddings and dropout
masks are the same whichever split executes them (R15).
"""

from __future__ import annotations

import numpy as np
from scipy.special import erf

F = np.float64


def round_bf16(x):
    """Storage precision of bf16 graphs (DESIGN.md D-TOL):
    the value a kernel that computes in fp32 stores as bf16 — fp64 -> nearest fp32
    -> nearest bf16 (round to nearest, ties to even on the 16 dropped bits).
    Returned widened to fp64."""
    b = np.ascontiguousarray(np.asarray(x, np.float64).astype(np.float32)).view(np.uint32).astype(np.uint64)
    b = (b + np.uint64(0x7FFF) + ((b >> np.uint64(16)) & np.uint64(1))) & np.uint64(0xFFFF0000)
    return b.astype(np.uint32).view(np.float32).astype(F)


# ---------------------------------------------------------------------------
# Philox4x32-10 counter-based RNG (Salmon et al., SC'11), SURVEY.md §8(c) R15,
# DESIGN.md reading D-RNG.  Element idx draws the 16-bit half (idx & 1, low half
# first) of word ((idx >> 1) & 3) of Philox(counter = (c_lo, c_hi, step, 0),
# key = (seed, 0x5453504C)) with c = idx >> 3 (one Philox call feeds eight
# consecutive elements), and keep = (half >= floor(p * 2^16)).  Pure integer
# maths, so both sides of the parity test take the identical keep/drop decision.
# ---------------------------------------------------------------------------
_M0, _M1 = np.uint64(0xD2511F53), np.uint64(0xCD9E8D57)
_W0, _W1 = 0x9E3779B9, 0xBB67AE85
_MASK32 = np.uint64(0xFFFFFFFF)
PHILOX_KEY1 = 0x5453504C


def philox4x32_10(c, k0, k1):
    """Philox4x32-10 on a tuple of four uint64 arrays holding 32-bit counters."""
    c0, c1, c2, c3 = c
    k0, k1 = k0 & 0xFFFFFFFF, k1 & 0xFFFFFFFF
    for r in range(10):
        p0 = _M0 * c0
        p1 = _M1 * c2
        hi0, lo0 = p0 >> np.uint64(32), p0 & _MASK32
        hi1, lo1 = p1 >> np.uint64(32), p1 & _MASK32
        c0, c1, c2, c3 = (hi1 ^ c1 ^ np.uint64(k0)), lo1, (hi0 ^ c3 ^ np.uint64(k1)), lo0
        k0 = (k0 + _W0) & 0xFFFFFFFF
        k1 = (k1 + _W1) & 0xFFFFFFFF
    return c0, c1, c2, c3


def philox_word(idx: np.ndarray, seed: int, step: int = 0) -> np.ndarray:
    """The 16-bit random draw of element idx (see above)."""
    idx = idx.astype(np.uint64)
    ctr = idx >> np.uint64(3)
    c0 = ctr & _MASK32
    c1 = ctr >> np.uint64(32)
    c2 = np.full_like(c0, np.uint64(step & 0xFFFFFFFF))
    c3 = np.zeros_like(c0)
    words = np.stack(philox4x32_10((c0, c1, c2, c3), seed, PHILOX_KEY1))
    w = words[((idx >> np.uint64(1)) & np.uint64(3)).astype(np.int64), np.arange(idx.shape[0])]
    return (w >> (np.uint64(16) * (idx & np.uint64(1)))) & np.uint64(0xFFFF)


def dropout_keep(shape, elem0: int, p: float, seed: int, step: int = 0) -> np.ndarray:
    n = int(np.prod(shape))
    w = philox_word(np.arange(elem0, elem0 + n, dtype=np.uint64), seed, step)
    thr = np.uint64(min(int(np.floor(p * 65536.0)), 65535))
    return (w >= thr).reshape(shape)


# ---------------------------------------------------------------------------
# Forward / backward of each op kind.  Arrays are fp64.
# ---------------------------------------------------------------------------

def linear_fwd(x, w, b):
    return x @ w.T + b


def linear_bwd(dy, x, w):
    """dX = dY W, dW = dY^T X, db = sum_rows dY."""
    return dy @ w, dy.T @ x, dy.sum(axis=0)


def relu_fwd(x):
    return np.maximum(x, 0.0)


def relu_bwd(dy, y):
    return dy * (y > 0)


def gelu_fwd(x):
    return 0.5 * x * (1.0 + erf(x / np.sqrt(2.0)))


def gelu_bwd(dy, x):
    cdf = 0.5 * (1.0 + erf(x / np.sqrt(2.0)))
    pdf = np.exp(-0.5 * x * x) / np.sqrt(2.0 * np.pi)
    return dy * (cdf + x * pdf)


def tanh_fwd(x):
    return np.tanh(x)


def tanh_bwd(dy, y):
    return dy * (1.0 - y * y)


def layernorm_fwd(x, g, b, eps):
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    xhat = (x - mu) / np.sqrt(var + eps)
    return xhat * g + b


def layernorm_bwd(dy, x, g, eps):
    """Returns dX, dgamma, dbeta (biased variance, per-row statistics)."""
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)
    rstd = 1.0 / np.sqrt(var + eps)
    xhat = (x - mu) * rstd
    dxhat = dy * g
    dx = rstd * (dxhat - dxhat.mean(axis=-1, keepdims=True)
                 - xhat * (dxhat * xhat).mean(axis=-1, keepdims=True))
    return dx, (dy * xhat).sum(axis=0), dy.sum(axis=0)


def add_fwd(a, b):
    return a + b


def dropout_fwd(x, p, seed, elem0, step=0):
    if p == 0.0:
        return x.copy()
    keep = dropout_keep(x.shape, elem0, p, seed, step)
    return np.where(keep, x / (1.0 - p), 0.0)


def dropout_bwd(dy, p, seed, elem0, step=0):
    return dropout_fwd(dy, p, seed, elem0, step)


def softmax_fwd(x, causal=False):
    """Row softmax over the last dim.  causal: x is [..., s, s] attention scores (query i,
    key j) and keys j > i are excluded (probability 0) — the decoder self-attention of the
    encoder-decoder Transformer."""
    if causal:
        s = x.shape[-1]
        x = np.where(np.triu(np.ones((s, s), bool), 1), -np.inf, x)
    m = x.max(axis=-1, keepdims=True)
    e = np.exp(x - m)
    return e / e.sum(axis=-1, keepdims=True)


def softmax_bwd(dy, y):
    return y * (dy - (dy * y).sum(axis=-1, keepdims=True))


def _heads(x, heads, seq):
    """[nb*s, h] -> [nb, a, s, d]."""
    nb = x.shape[0] // seq
    return x.reshape(nb, seq, heads, -1).transpose(0, 2, 1, 3)


def _merge(xh):
    """[nb, a, s, d] -> [nb*s, h]."""
    nb, a, s, d = xh.shape
    return xh.transpose(0, 2, 1, 3).reshape(nb * s, a * d)


def attn_qk_fwd(q, k, heads, seq, alpha):
    return alpha * (_heads(q, heads, seq) @ _heads(k, heads, seq).transpose(0, 1, 3, 2))


def attn_qk_bwd(ds, q, k, heads, seq, alpha):
    qh, kh = _heads(q, heads, seq), _heads(k, heads, seq)
    dq = alpha * (ds @ kh)
    dk = alpha * (ds.transpose(0, 1, 3, 2) @ qh)
    return _merge(dq), _merge(dk)


def attn_pv_fwd(p, v, heads, seq):
    return _merge(p @ _heads(v, heads, seq))


def attn_pv_bwd(dc, p, v, heads, seq):
    dch = _heads(dc, heads, seq)
    vh = _heads(v, heads, seq)
    dp = dch @ vh.transpose(0, 1, 3, 2)
    dv = p.transpose(0, 1, 3, 2) @ dch
    return dp, _merge(dv)


def attention_fwd(q, k, v, heads, seq, alpha, p, seed, elem0, step=0):
    """Fused attention micro-op (the composition of attn_qk,
    softmax, dropout and attn_pv, P:L119's attention block): C = dropout(softmax(
    alpha Q_h K_h^T)) V_h with heads merged, plus the row log-sum-exp
    lse[b,a,i] = log sum_j exp(S_ij) that its backward reads.  The dropout mask is the
    unfused op's: Philox on the element index of the [b,a,s,s] probabilities
    (elem0 = first sample's offset there), so fused and unfused graphs compute the
    same function.  Returns (C, lse, mask words)."""
    s = attn_qk_fwd(q, k, heads, seq, alpha)
    m = s.max(axis=-1, keepdims=True)
    lse = (m + np.log(np.exp(s - m).sum(axis=-1, keepdims=True)))[..., 0]
    pd = dropout_fwd(softmax_fwd(s), p, seed, elem0, step)
    return attn_pv_fwd(pd, v, heads, seq), lse, attention_mask_words(s.shape, p, seed, elem0, step)


def attention_mask_words(shape, p, seed, elem0, step=0):
    """The keep mask of attention_fwd packed 32 keys per int32 word, key 32w + j at bit j
    ([b,a,s,s/32]); all ones when p = 0.  The fused op stores it for its backward."""
    keep = np.ones(shape, bool) if p == 0.0 else dropout_keep(shape, elem0, p, seed, step)
    nw = (shape[-1] + 31) // 32  # keys past the end read as dropped bits 0
    keep = np.concatenate([keep, np.zeros(shape[:-1] + (nw * 32 - shape[-1],), bool)], axis=-1)
    bits = keep.reshape(shape[:-1] + (nw, 32)).astype(np.uint64)
    w = (bits << np.arange(32, dtype=np.uint64)).sum(axis=-1)
    return w.astype(np.uint32).view(np.int32)


def attention_bwd(dc, q, k, v, heads, seq, alpha, p, seed, elem0, step=0):
    """VJP of attention_fwd w.r.t. Q, K, V: the chain rule through the same four ops."""
    pr = softmax_fwd(attn_qk_fwd(q, k, heads, seq, alpha))
    pd = dropout_fwd(pr, p, seed, elem0, step)
    dpd, dv = attn_pv_bwd(dc, pd, v, heads, seq)
    ds = softmax_bwd(dropout_bwd(dpd, p, seed, elem0, step), pr)
    dq, dk = attn_qk_bwd(ds, q, k, heads, seq, alpha)
    return dq, dk, dv


def embed_fwd(ids, tt, wword, wpos, wtype, seq, row0):
    pos = (np.arange(row0, row0 + ids.shape[0]) % seq)
    return wword[ids] + wpos[pos] + wtype[tt]


def embed_bwd(dy, ids, tt, seq, row0, shapes):
    dword = np.zeros(shapes[0], F)
    dpos = np.zeros(shapes[1], F)
    dtype_ = np.zeros(shapes[2], F)
    pos = (np.arange(row0, row0 + ids.shape[0]) % seq)
    np.add.at(dword, ids, dy)
    np.add.at(dpos, pos, dy)
    np.add.at(dtype_, tt, dy)
    return dword, dpos, dtype_


def cls_fwd(x, seq):
    return x[::seq].copy()


def cls_bwd(dy, seq, rows):
    dx = np.zeros((rows, dy.shape[1]), F)
    dx[::seq] = dy
    return dx


def xent_fwd(z, labels, b_global):
    """Sum over this block of (logsumexp(z) - z[label]) / B_global (R14)."""
    m = z.max(axis=1, keepdims=True)
    lse = (m + np.log(np.exp(z - m).sum(axis=1, keepdims=True)))[:, 0]
    return float((lse - z[np.arange(z.shape[0]), labels]).sum() / b_global)


def xent_bwd(z, labels, b_global):
    dz = softmax_fwd(z)
    dz[np.arange(z.shape[0]), labels] -= 1.0
    return dz / b_global


# ---------------------------------------------------------------------------
# CNN ops (configs 2-3).  NHWC activations, KRSC weights; conv via im2col.
# ---------------------------------------------------------------------------

def _im2col(x, R, S, stride, pad):
    """x [N,H,W,C] -> cols [N,P,Q,R,S,C] (zero padding)."""
    N, H, W, C = x.shape
    P = (H + 2 * pad - R) // stride + 1
    Q = (W + 2 * pad - S) // stride + 1
    xp = np.pad(x, ((0, 0), (pad, pad), (pad, pad), (0, 0)))
    cols = np.empty((N, P, Q, R, S, C), x.dtype)
    for r in range(R):
        for s in range(S):
            cols[:, :, :, r, s, :] = xp[:, r:r + stride * P:stride, s:s + stride * Q:stride, :]
    return cols


def conv2d_fwd(x, w, b, stride, pad):
    """Y[n,p,q,k] = sum_{r,s,c} X[n, p*st+r-pad, q*st+s-pad, c] W[k,r,s,c] (+ b[k])."""
    K, R, S, C = w.shape
    cols = _im2col(x, R, S, stride, pad)
    N, P, Q = cols.shape[:3]
    y = cols.reshape(N * P * Q, R * S * C) @ w.reshape(K, R * S * C).T
    if b is not None:
        y = y + b
    return y.reshape(N, P, Q, K)


def conv2d_bwd(dy, x, w, stride, pad):
    """dX (col2im of dY W), dW = dY^T cols, db = sum dY."""
    K, R, S, C = w.shape
    N, H, W_, _ = x.shape
    cols = _im2col(x, R, S, stride, pad)
    _, P, Q = cols.shape[:3]
    dy2 = dy.reshape(N * P * Q, K)
    dw = (dy2.T @ cols.reshape(N * P * Q, R * S * C)).reshape(K, R, S, C)
    dcols = (dy2 @ w.reshape(K, R * S * C)).reshape(N, P, Q, R, S, C)
    dxp = np.zeros((N, H + 2 * pad, W_ + 2 * pad, C), F)
    for r in range(R):
        for s in range(S):
            dxp[:, r:r + stride * P:stride, s:s + stride * Q:stride, :] += dcols[:, :, :, r, s, :]
    dx = dxp[:, pad:pad + H, pad:pad + W_, :]
    return dx, dw, dy2.sum(axis=0)


def batchnorm_fwd(x, g, b, eps):
    """Train-mode BN over (N,H,W) per channel, biased variance."""
    mu = x.mean(axis=(0, 1, 2))
    var = ((x - mu) ** 2).mean(axis=(0, 1, 2))
    return (x - mu) / np.sqrt(var + eps) * g + b


def batchnorm_bwd(dy, x, g, eps):
    mu = x.mean(axis=(0, 1, 2))
    var = ((x - mu) ** 2).mean(axis=(0, 1, 2))
    rstd = 1.0 / np.sqrt(var + eps)
    xhat = (x - mu) * rstd
    dxhat = dy * g
    m = x.shape[0] * x.shape[1] * x.shape[2]
    dx = rstd * (dxhat - dxhat.sum(axis=(0, 1, 2)) / m - xhat * (dxhat * xhat).sum(axis=(0, 1, 2)) / m)
    return dx, (dy * xhat).sum(axis=(0, 1, 2)), dy.sum(axis=(0, 1, 2))


def maxpool_fwd(x, k, stride, pad):
    """Max over k x k windows; padding never wins (-inf)."""
    N, H, W, C = x.shape
    P = (H + 2 * pad - k) // stride + 1
    Q = (W + 2 * pad - k) // stride + 1
    xp = np.pad(x, ((0, 0), (pad, pad), (pad, pad), (0, 0)), constant_values=-np.inf)
    y = np.full((N, P, Q, C), -np.inf)
    for r in range(k):
        for s in range(k):
            y = np.maximum(y, xp[:, r:r + stride * P:stride, s:s + stride * Q:stride, :])
    return y


def maxpool_bwd(dy, x, k, stride, pad):
    """Gradient to the first maximum in row-major window order."""
    N, H, W, C = x.shape
    P, Q = dy.shape[1], dy.shape[2]
    xp = np.pad(x, ((0, 0), (pad, pad), (pad, pad), (0, 0)), constant_values=-np.inf)
    y = maxpool_fwd(x, k, stride, pad)
    taken = np.zeros(dy.shape, bool)
    dxp = np.zeros(xp.shape, F)
    for r in range(k):
        for s in range(k):
            win = xp[:, r:r + stride * P:stride, s:s + stride * Q:stride, :]
            hit = (win == y) & ~taken
            dxp[:, r:r + stride * P:stride, s:s + stride * Q:stride, :] += np.where(hit, dy, 0.0)
            taken |= hit
    return dxp[:, pad:pad + H, pad:pad + W, :]


def avgpool_fwd(x):
    """Global average pool [N,H,W,C] -> [N,C]."""
    return x.mean(axis=(1, 2))


def avgpool_bwd(dy, shape):
    N, H, W, C = shape
    return np.broadcast_to(dy[:, None, None, :] / (H * W), shape).copy()


def batchnorm_stats(x):
    """Full-batch mean and biased variance per channel of x [...,C]."""
    ax = tuple(range(x.ndim - 1))
    mu = x.mean(axis=ax)
    return mu, ((x - mu) ** 2).mean(axis=ax)


def batchnorm_fwd_with(x, g, b, mu, var, eps):
    """Normalise a block of samples with the full-batch statistics (R13)."""
    return (x - mu) / np.sqrt(var + eps) * g + b


def batchnorm_bwd_sums(dy, x, g, mu, var, eps):
    """Full-batch sums for the BN backward: sum(dy*g), sum(dy*g*xhat), dgamma, dbeta."""
    ax = tuple(range(x.ndim - 1))
    xhat = (x - mu) / np.sqrt(var + eps)
    return (dy * g).sum(axis=ax), (dy * g * xhat).sum(axis=ax), (dy * xhat).sum(axis=ax), dy.sum(axis=ax)


def batchnorm_bwd_with(dy, x, g, mu, var, s1, s2, m, eps):
    rstd = 1.0 / np.sqrt(var + eps)
    xhat = (x - mu) * rstd
    return rstd * (dy * g - s1 / m - xhat * s2 / m)
