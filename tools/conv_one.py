"""Launch one conv micro-op kernel a few times (for ncu captures).
    python tools/conv_one.py MODE n H W C K R S stride pad"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402

mode = int(sys.argv[1])
n, H, W, C, K, R, S, st, pad = (int(v) for v in sys.argv[2:11])
P, Q = (H + 2 * pad - R) // st + 1, (W + 2 * pad - S) // st + 1
bf = torch.bfloat16
x = torch.randn(n, H, W, C, device="cuda", dtype=bf)
w = torch.randn(K, R, S, C, device="cuda", dtype=bf)
dy = torch.randn(n, P, Q, K, device="cuda", dtype=bf)
out = {1: torch.empty(n, P, Q, K, device="cuda", dtype=bf), 2: torch.empty_like(x),
       3: torch.empty(K, R, S, C, device="cuda", dtype=torch.float32)}[mode]
for _ in range(3):
    tsplit.conv2d(mode, (n, H, W, C, K, R, S, st, pad), x, w, dy, out)
torch.cuda.synchronize()
