"""Per-shape throughput of the tcgen05 GEMM (C ABI) vs cuBLAS (torch.matmul) for
the BERT-Large micro-op GEMM forms.  Usage: python tools/gemm_bench.py"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402

T, H, F = 16384, 1024, 4096


def timeit(fn, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps / 1e3


def case(name, M, N, K, ta, tb, out="bf16", batch=1, beta=0.0):
    A = torch.randn(batch, *( (K, M) if ta else (M, K) ), device="cuda").to(torch.bfloat16)
    B = torch.randn(batch, *( (K, N) if tb else (N, K) ), device="cuda").to(torch.bfloat16)
    od = torch.float32 if out == "f32" else torch.bfloat16
    C = torch.zeros(batch, M, N, device="cuda", dtype=od)
    lda, ldb = (M if ta else K), (N if tb else K)
    L = tsplit.lib()
    st = torch.cuda.current_stream().cuda_stream

    def ours():
        tsplit.check(L.ts_gemm_bf16(M, N, K, batch, A.data_ptr(), lda, A[0].numel(), ta, B.data_ptr(), ldb,
                                    B[0].numel(), tb, C.data_ptr(), N, M * N, 0 if out == "f32" else 1, 1.0, beta,
                                    None, st))
    Aop = A.transpose(1, 2) if ta else A
    Bop = B if tb else B.transpose(1, 2)

    def cublas():
        torch.matmul(Aop, Bop, out=C if out == "bf16" else None) if out == "bf16" else torch.matmul(Aop, Bop)
    fl = 2.0 * M * N * K * batch
    modes = {}
    all_modes = ((1, "cta1"), (5, "cta1_nosplit"), (2, "pair"), (6, "pair_nosplit"), (0, "auto"))
    only = os.environ.get("MODES")  # e.g. MODES=0 (ncu captures of the cost model's choice)
    for mode, tag in all_modes:
        if only is not None and str(mode) not in only.split(","):
            continue
        tsplit.check(L.ts_gemm_set_mode(mode))
        t = timeit(ours)
        cfg = (tsplit.C.c_int32 * 8)()
        tsplit.check(L.ts_gemm_last_config(cfg))
        modes[tag] = {"tflops": fl / t / 1e12, "us": t * 1e6, "bn": cfg[0], "cg": cfg[1], "ksplit": cfg[2],
                      "units": cfg[3], "pair_slots": cfg[5], "split_from": cfg[6]}
    tsplit.check(L.ts_gemm_set_mode(0))
    t_ours = modes[next(iter(modes))]["us"] / 1e6
    t_cub = timeit(cublas)
    r = {"name": name, "M": M, "N": N, "K": K, "batch": batch, "ta": ta, "tb": tb, "out": out,
         "ours_tflops": fl / t_ours / 1e12, "cublas_tflops": fl / t_cub / 1e12, "ours_us": t_ours * 1e6,
         "modes": modes}
    print(json.dumps(r), flush=True)
    return r


if __name__ == "__main__":
    res = []
    res.append(case("qkv/proj fwd", T, H, H, 0, 0))
    res.append(case("ffn1 fwd", T, F, H, 0, 0))
    res.append(case("ffn2 fwd", T, H, F, 0, 0))
    res.append(case("proj dX", T, H, H, 0, 1))
    res.append(case("ffn1 dX", T, H, F, 0, 1))
    res.append(case("ffn2 dX", T, F, H, 0, 1))
    res.append(case("proj dW", H, H, T, 1, 1, out="f32", beta=1.0))
    res.append(case("ffn1 dW", F, H, T, 1, 1, out="f32", beta=1.0))
    res.append(case("ffn2 dW", H, F, T, 1, 1, out="f32", beta=1.0))
    res.append(case("p=4 ffn1 fwd", T // 4, F, H, 0, 0))
    res.append(case("qkv dW grouped-size", 3 * H, H, T, 1, 1, out="f32", beta=1.0))
    res.append(case("p=2 qkv fwd", T // 2, H, H, 0, 0))
    res.append(case("p=4 qkv fwd", T // 4, H, H, 0, 0))
    res.append(case("p=4 ffn2 fwd", T // 4, H, F, 0, 0))
    res.append(case("attn QK^T", 512, 512, 64, 0, 0, batch=512))
    res.append(case("attn PV", 512, 64, 512, 0, 1, batch=512))
    res.append(case("attn dS^T Q", 512, 64, 512, 1, 1, batch=512))
    json.dump(res, open(os.environ.get("OUT", "gpurun_out/gemm_bench.json"), "w"), indent=1)
