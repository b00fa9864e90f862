"""Bias-gradient column sums ([rows, N] bf16 -> fp32 [N]) at the BERT-Large shapes: time
(CUDA events) and HBM GB/s of the input read.   python tools/colsum_bench.py"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402

res = []
for rows, n in ((16384, 1024), (16384, 4096), (8192, 1024), (4096, 4096)):
    x = torch.randn(rows, n, device="cuda").to(torch.bfloat16)
    out = torch.zeros(n, device="cuda")
    ws = torch.zeros(256 * 2 * 4096 + 1024, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for _ in range(3):
        tsplit.column_sum(x, out, ws)
    ts = []
    for _ in range(20):
        flush.zero_()  # a cold input, as in the step (written by another kernel long before)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        tsplit.column_sum(x, out, ws)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    ts.sort()
    us = ts[len(ts) // 2]
    err = float((out.double() - x.double().sum(0)).abs().max() / x.double().sum(0).abs().max())
    res.append({"rows": rows, "n": n, "us": us, "gbs": rows * n * 2 / us / 1e3, "rel_err": err})
    print(json.dumps(res[-1]), flush=True)
