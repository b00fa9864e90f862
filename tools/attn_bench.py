"""Time the fused-attention kernels (forward; backward = dQ + dK/dV kernels) at a given shape with
CUDA events on the launching stream.  python tools/attn_bench.py [nb heads seq p] -> JSON line.
FLOP counted: forward 2 products (QK^T, PV) = 4*nb*heads*seq^2*d; backward 5 products
(S, dP, dV, dK, dQ) = 10*nb*heads*seq^2*d (the dQ kernel's recomputed S, dP are not credited)."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402

nb, heads, seq = (int(v) for v in sys.argv[1:4]) if len(sys.argv) > 3 else (32, 16, 512)
p = float(sys.argv[4]) if len(sys.argv) > 4 else 0.1
d = 64
torch.manual_seed(0)
Q = torch.randn(nb * seq, heads * d, device="cuda", dtype=torch.bfloat16)
K, V, DC = torch.randn_like(Q), torch.randn_like(Q), torch.randn_like(Q)
C = torch.empty_like(Q)
L = torch.empty(nb, heads, seq, device="cuda")
M = torch.empty(nb, heads, seq, seq // 32, device="cuda", dtype=torch.int32)
ws = torch.empty(nb * heads * seq, device="cuda")
dq, dk, dv = torch.empty_like(Q), torch.empty_like(Q), torch.empty_like(Q)
g = (nb, heads, seq, d, 1, 0, 0)


def fwd():
    return tsplit.attention(1, g, 0.125, p, Q, K, V, c=C, lse=L, mask=M)


def bwd():
    return tsplit.attention(2, g, 0.125, p, Q, K, V, c=C, lse=L, mask=M, dc=DC, dq=dq, dk=dk, dv=dv, ws=ws)


def timeit(fn, n=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(n):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / n * 1e3


path = fwd()
tf = timeit(fwd)
tb = timeit(bwd)
base = nb * heads * seq * seq * d
print(json.dumps({"shape": [nb, heads, seq, d], "p": p, "path": path, "fwd_us": tf, "bwd_us": tb,
                  "fwd_tflops": 4 * base / tf / 1e6, "bwd_tflops": 10 * base / tb / 1e6}))
