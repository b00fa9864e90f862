"""Time the fused GELU-epilogue GEMMs (ts_gemm_bf16_epi) against the plain product of the same
shape (ts_gemm_bf16), CUDA events on the launching stream.
    python tools/gemm_epi_bench.py [M N K]   (default: BERT-Large FFN1 16384 4096 1024) -> JSON lines"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402

M, N, K = (int(v) for v in sys.argv[1:4]) if len(sys.argv) > 3 else (16384, 4096, 1024)
L = tsplit.lib()
A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
B = torch.randn(N, K, device="cuda").to(torch.bfloat16) * 0.03
bias = torch.randn(N, device="cuda").to(torch.bfloat16)
U, H = (torch.empty(M, N, device="cuda", dtype=torch.bfloat16) for _ in range(2))


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


forms = {
    "plain": lambda: tsplit.check(L.ts_gemm_bf16(M, N, K, 1, A.data_ptr(), K, 0, 0, B.data_ptr(), K, 0, 0,
                                                 U.data_ptr(), N, 0, 1, 1.0, 0.0, bias.data_ptr(), None)),
    "gelu_fwd": lambda: tsplit.check(L.ts_gemm_bf16_epi(1, M, N, K, A.data_ptr(), K, 0, B.data_ptr(), K, 0,
                                                        U.data_ptr(), N, 1.0, bias.data_ptr(), H.data_ptr(), N, None)),
    "gelu_bwd": lambda: tsplit.check(L.ts_gemm_bf16_epi(2, M, N, K, A.data_ptr(), K, 0, B.data_ptr(), K, 0,
                                                        H.data_ptr(), N, 1.0, None, U.data_ptr(), N, None)),
}
only = sys.argv[4].split(",") if len(sys.argv) > 4 else list(forms)
for name in only:
    us = timeit(forms[name])
    print(json.dumps({"form": name, "M": M, "N": N, "K": K, "us": us, "tflops": 2.0 * M * N * K / us / 1e6}))
