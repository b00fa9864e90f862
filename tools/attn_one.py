"""Launch the fused-attention forward once (debug / ncu).  python tools/attn_one.py nb heads seq p [mode]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402

nb, heads, seq = (int(v) for v in sys.argv[1:4])
p = float(sys.argv[4])
mode = int(sys.argv[5]) if len(sys.argv) > 5 else 1
d = 64
Q = torch.randn(nb * seq, heads * d, device="cuda", dtype=torch.bfloat16)
K, V, DC = torch.randn_like(Q), torch.randn_like(Q), torch.randn_like(Q)
C = torch.empty_like(Q)
L = torch.empty(nb, heads, seq, device="cuda")
M = torch.empty(nb, heads, seq, seq // 32, device="cuda", dtype=torch.int32)
ws = torch.empty(nb * heads * seq, device="cuda")
dq, dk, dv = torch.empty_like(Q), torch.empty_like(Q), torch.empty_like(Q)
g = (nb, heads, seq, d, 1, 0, 0)
for _ in range(3):
    used = tsplit.attention(1, g, 0.125, p, Q, K, V, c=C, lse=L, mask=M)
    if mode == 2:
        tsplit.attention(2, g, 0.125, p, Q, K, V, c=C, lse=L, mask=M, dc=DC, dq=dq, dk=dk, dv=dv, ws=ws)
torch.cuda.synchronize()
print("ok path", used, float(C.float().abs().mean()))
