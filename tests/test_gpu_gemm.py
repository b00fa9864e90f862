"""tcgen05/TMA GEMM and SIMT GEMM through the C ABI vs a plain fp32 PyTorch
reference of the same product (operands are the exact bf16 values, upcast)."""

import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_niemyc22_b200 import tsplit  # noqa: E402


def _mk(shape, dtype=torch.bfloat16, seed=0):
    g = torch.Generator(device="cuda").manual_seed(seed)
    return torch.randn(*shape, generator=g, device="cuda", dtype=torch.float32).to(dtype)


def _op(x, mn):
    """Logical [rows, K] operand stored K-major (x) or MN-major (x^T stored)."""
    return x.t().contiguous() if mn else x.contiguous()


CASES = [
    # M, N, K, batch, ta, tb, out
    (256, 256, 128, 1, 0, 0, "bf16"),
    (512, 1024, 1024, 1, 0, 0, "bf16"),
    (384, 192, 320, 1, 0, 1, "bf16"),
    (256, 320, 192, 1, 1, 1, "f32"),
    (200, 136, 72, 1, 0, 0, "bf16"),     # ragged M/N/K
    (136, 64, 96, 3, 1, 0, "f32"),       # ragged + batched (MN-major ld must be 16 B aligned)
    (512, 64, 512, 4, 0, 1, "bf16"),     # attention P.V shape
    (1024, 4096, 1024, 1, 0, 0, "bf16"),
    (1024, 1024, 4096, 1, 1, 1, "f32"),  # dW shape
]


@pytest.mark.parametrize("M,N,K,batch,ta,tb,out", CASES)
def test_gemm_tc_matches_torch(M, N, K, batch, ta, tb, out):
    torch.cuda.synchronize()
    A = [_mk((M, K), seed=1 + b) for b in range(batch)]
    B = [_mk((N, K), seed=100 + b) for b in range(batch)]
    As = torch.stack([_op(a, ta) for a in A])
    Bs = torch.stack([_op(b, tb) for b in B])
    od = torch.float32 if out == "f32" else torch.bfloat16
    Cc = torch.zeros(batch, M, N, device="cuda", dtype=od)
    lda = M if ta else K
    ldb = N if tb else K
    st = tsplit.lib().ts_gemm_bf16(M, N, K, batch, As.data_ptr(), lda, As[0].numel(), ta, Bs.data_ptr(), ldb,
                                   Bs[0].numel(), tb, Cc.data_ptr(), N, M * N, 0 if out == "f32" else 1,
                                   1.0, 0.0, None, None)
    tsplit.check(st)
    torch.cuda.synchronize()
    for b in range(batch):
        ref = A[b].float() @ B[b].float().t()
        got = Cc[b].float()
        err = ((got - ref).norm() / ref.norm()).item()
        assert err < (1e-5 if out == "f32" else 8e-3), (b, err)


def test_gemm_tc_alpha_beta_bias():
    M, N, K = 256, 384, 256
    A, B = _mk((M, K), seed=3), _mk((N, K), seed=4)
    bias = _mk((N,), seed=5)
    C0 = torch.randn(M, N, device="cuda")
    C = C0.clone()
    tsplit.check(tsplit.lib().ts_gemm_bf16(M, N, K, 1, A.data_ptr(), K, 0, 0, B.data_ptr(), K, 0, 0, C.data_ptr(), N,
                                           0, 0, 0.5, 1.0, bias.data_ptr(), None))
    torch.cuda.synchronize()
    ref = 0.5 * (A.float() @ B.float().t()) + bias.float() + C0
    assert ((C - ref).norm() / ref.norm()).item() < 1e-5


def test_gemm_simt_f32():
    M, N, K = 70, 33, 45
    A = torch.randn(K, M, device="cuda")  # MN-major
    B = torch.randn(N, K, device="cuda")
    C = torch.zeros(M, N, device="cuda")
    tsplit.check(tsplit.lib().ts_gemm_f32(M, N, K, A.data_ptr(), M, 1, B.data_ptr(), K, 0, C.data_ptr(), N, 1.0,
                                          0.0, None, None))
    torch.cuda.synchronize()
    ref = A.t().double() @ B.t().double()
    assert ((C.double() - ref).norm() / ref.norm()).item() < 1e-6


@pytest.mark.parametrize("M,N,K,out,beta", [
    (1024, 1024, 16384, "f32", 0.0),   # dW with split-K (reduce-add partials)
    (1024, 1024, 16384, "f32", 1.0),   # dW accumulated across splits (beta = 1)
    (256, 512, 640, "bf16", 1.0),      # activation-gradient accumulation in bf16
    (200, 72, 128, "f32", 1.0),        # ragged tile edges through the TMA store
])
def test_gemm_tc_accumulate_and_splitk(M, N, K, out, beta):
    A = _mk((K, M), seed=11)   # MN-major operands, as in dW = dY^T X
    B = _mk((K, N), seed=12)
    od = torch.float32 if out == "f32" else torch.bfloat16
    C0 = torch.randn(M, N, device="cuda").to(od)
    C = C0.clone()
    tsplit.check(tsplit.lib().ts_gemm_bf16(M, N, K, 1, A.data_ptr(), M, 0, 1, B.data_ptr(), N, 0, 1, C.data_ptr(), N,
                                           0, 0 if out == "f32" else 1, 1.0, beta, None, None))
    torch.cuda.synchronize()
    ref = A.double().t() @ B.double() + beta * C0.double()
    err = ((C.double() - ref).norm() / ref.norm()).item()
    # fp32 accumulation over K terms: ~sqrt(K) * 2^-24 relative
    assert err < (3e-5 if out == "f32" else 8e-3), err
