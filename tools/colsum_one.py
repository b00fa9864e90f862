"""One bias column sum [rows, n] (ncu captures).  python tools/colsum_one.py rows n"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402

rows, n = int(sys.argv[1]), int(sys.argv[2])
x = torch.randn(rows, n, device="cuda").to(torch.bfloat16)
out = torch.zeros(n, device="cuda")
ws = torch.zeros(256 * 2 * 4096 + 1024, device="cuda")
for _ in range(3):
    tsplit.column_sum(x, out, ws)
torch.cuda.synchronize()
print("ok")
