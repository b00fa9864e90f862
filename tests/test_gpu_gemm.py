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
    (300, 256, 192, 1, 0, 0, "bf16"),    # CTA pair: second CTA's rows partly past M
    (129, 384, 64, 2, 0, 1, "f32"),      # CTA pair: second CTA entirely past M
    (640, 128, 256, 1, 1, 0, "bf16"),    # pair tile width 128 (64 B rows per CTA)
    (4096, 1024, 1024, 1, 0, 0, "bf16"),  # BERT projection shape at p = 4
    (16384, 1024, 256, 1, 0, 0, "bf16"),  # 512 tiles: the tail wave runs as half-width units
    (16384, 1024, 128, 1, 0, 1, "bf16"),  # same, MN-major B
    (20000, 1024, 64, 1, 1, 1, "f32"),    # tail split with ragged M, both operands MN-major
]


def _cfg():
    out = (tsplit.C.c_int32 * 8)()
    tsplit.check(tsplit.lib().ts_gemm_last_config(out))
    return list(out)


@pytest.fixture
def gemm_mode():
    yield lambda m: tsplit.check(tsplit.lib().ts_gemm_set_mode(m))
    tsplit.check(tsplit.lib().ts_gemm_set_mode(0))


@pytest.mark.parametrize("mode", [0, 1, 2])
@pytest.mark.parametrize("M,N,K,batch,ta,tb,out", CASES)
def test_gemm_tc_matches_torch(M, N, K, batch, ta, tb, out, mode, gemm_mode):
    """mode 1 = single-CTA tiles, 2 = CTA-pair (tcgen05 cta_group::2) tiles, 0 = cost model."""
    gemm_mode(mode)
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
    cfg = _cfg()
    if mode:
        assert cfg[1] == (2 if mode == 2 and M > 128 and N > 64 else 1), cfg
        if M >= 16384 and N == 1024:  # 512 (resp. 256 pair) tiles: tail wave split in halves
            assert cfg[6] < cfg[3], cfg
    for b in range(batch):
        ref = A[b].float() @ B[b].float().t()
        got = Cc[b].float()
        err = ((got - ref).norm() / ref.norm()).item()
        assert err < (1e-5 if out == "f32" else 8e-3), (b, err)


@pytest.mark.parametrize("mode", [1, 2])
def test_gemm_tc_alpha_beta_bias(mode, gemm_mode):
    gemm_mode(mode)
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


@pytest.mark.parametrize("M,N,K", [(70, 33, 45), (32, 2, 1024), (2, 1024, 32), (4, 3, 4096)])
def test_gemm_simt_f32(M, N, K):
    """CUDA-core paths: the tiled kernel, and the warp-per-output kernel for tiny outputs with
    a long reduction (the 2-class classifier of BERT: 32 x 2 x 1024)."""
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
@pytest.mark.parametrize("mode", [1, 2])
def test_gemm_tc_accumulate_and_splitk(M, N, K, out, beta, mode, gemm_mode):
    gemm_mode(mode)
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


def _ptrs(ts):
    return (tsplit.C.c_void_p * len(ts))(*[t.data_ptr() for t in ts])


@pytest.mark.parametrize("mode", [0, 1, 2])
@pytest.mark.parametrize("gdim,M,N,K,ta,tb,out,beta", [
    (1, 1024, 3 * 256, 256, 0, 0, "bf16", 0.0),    # q/k/v forward: shared X, per-group W, C, bias
    (1, 600, 3 * 512, 192, 0, 0, "bf16", 0.0),     # ragged M
    (2, 1024, 256, 3 * 256, 0, 1, "bf16", 1.0),    # q/k/v dX: sum over groups into one C (accumulate)
    (2, 640, 384, 3 * 128, 0, 1, "bf16", 0.0),
    (3, 3 * 256, 256, 2048, 1, 1, "f32", 1.0),     # q/k/v dW: per-group dY^T, shared X, per-group dW
    (3, 3 * 512, 512, 1024, 1, 1, "f32", 0.0),
    (1, 512, 3 * 96, 128, 0, 0, "bf16", 0.0),      # N/groups = 96: no grouped tiling, per-group fallback
    (3, 3 * 64, 256, 512, 1, 1, "f32", 1.0),       # M/groups = 64: per-group fallback
])
def test_gemm_tc_grouped(gdim, M, N, K, ta, tb, out, beta, mode, gemm_mode):
    """Grouped product = the per-group plain products (fp32 torch reference)."""
    gemm_mode(mode)
    G = 3
    Mg, Ng, Kg = (M // G if gdim == 3 else M), (N // G if gdim == 1 else N), (K // G if gdim == 2 else K)
    A = [_mk((Mg, Kg), seed=1 + i) for i in range(G if gdim != 1 else 1)]
    B = [_mk((Ng, Kg), seed=10 + i) for i in range(G if gdim != 3 else 1)]
    od = torch.float32 if out == "f32" else torch.bfloat16
    nC = G if gdim != 2 else 1
    Cs = [torch.randn(Mg, Ng, device="cuda").to(od) for _ in range(nC)]
    C0 = [c.clone() for c in Cs]
    bias = [_mk((Ng,), seed=40 + i) for i in range(G if gdim == 1 else 1)] if gdim == 1 else None
    Aop = [_op(a, ta) for a in A]
    Bop = [_op(b, tb) for b in B]
    lda = Mg if ta else Kg
    ldb = Ng if tb else Kg
    st = tsplit.lib().ts_gemm_bf16_grouped(G, gdim, M, N, K, _ptrs(Aop), lda, ta, _ptrs(Bop), ldb, tb, _ptrs(Cs), Ng,
                                           0 if out == "f32" else 1, 1.0, beta, _ptrs(bias) if bias else None, None)
    tsplit.check(st)
    torch.cuda.synchronize()
    for i in range(nC):
        if gdim == 1:
            ref = A[0].float() @ B[i].float().t() + bias[i].float()
        elif gdim == 2:
            ref = sum(A[j].float() @ B[j].float().t() for j in range(G))
        else:
            ref = A[i].float() @ B[0].float().t()
        ref = ref + beta * C0[i].float()
        err = ((Cs[i].float() - ref).norm() / ref.norm()).item()
        assert err < (2e-5 if out == "f32" else 8e-3), (i, err)


@pytest.mark.parametrize("rows,n", [(16384, 1024), (16384, 4096), (100, 24), (4096, 8), (77, 1000)])
@pytest.mark.parametrize("dtype", ["bf16", "f32"])
def test_bias_column_sum(rows, n, dtype):
    """Bias-gradient column sums (ts_row_op 0): fp32 result within fp32 summation error of
    the fp64 sum, deterministic across calls, accumulate flag."""
    dt = torch.bfloat16 if dtype == "bf16" else torch.float32
    x = torch.randn(rows, n, device="cuda").to(dt)
    out = torch.zeros(n, device="cuda")
    ws = torch.zeros(256 * 2 * 4096 + 1024, device="cuda")
    tsplit.column_sum(x, out, ws)
    torch.cuda.synchronize()
    ref = x.double().sum(0)
    scale = x.double().abs().sum(0).max()
    assert float((out.double() - ref).abs().max() / scale) < 1e-6
    again = torch.zeros(n, device="cuda")
    tsplit.column_sum(x, again, ws)
    tsplit.column_sum(x, again, ws, acc=1)
    torch.cuda.synchronize()
    assert torch.equal(2 * out, again) or float((again.double() - 2 * ref).abs().max() / scale) < 2e-6


@pytest.mark.parametrize("mode", [0, 1, 2])
@pytest.mark.parametrize("M,N,K", [(1024, 4096, 1024), (384, 1024, 4096), (256, 192, 320)])
def test_gemm_tc_fused_gelu_epilogues(M, N, K, mode, gemm_mode):
    """ts_gemm_bf16_epi (reading D-FUSE): epi 1 writes U = A B^T + bias and gelu(bf16(U));
    epi 2 writes dU = bf16(A B^T) * gelu'(U) — against torch's exact erf GELU in fp32."""
    gemm_mode(mode)
    A, B, bias = _mk((M, K), seed=3), _mk((N, K), seed=4), _mk((N,), seed=5)
    U = torch.empty(M, N, device="cuda", dtype=torch.bfloat16)
    H = torch.empty_like(U)
    tsplit.check(tsplit.lib().ts_gemm_bf16_epi(1, M, N, K, A.data_ptr(), K, 0, B.data_ptr(), K, 0, U.data_ptr(), N,
                                               1.0, bias.data_ptr(), H.data_ptr(), N, None))
    torch.cuda.synchronize()
    u_ref = A.float() @ B.float().t() + bias.float()
    assert ((U.float() - u_ref).norm() / u_ref.norm()).item() < 8e-3
    h_ref = torch.nn.functional.gelu(U.float())  # from the stored bf16 U, as the kernel does
    assert ((H.float() - h_ref).norm() / h_ref.norm()).item() < 8e-3
    dU = torch.empty_like(U)
    tsplit.check(tsplit.lib().ts_gemm_bf16_epi(2, M, N, K, A.data_ptr(), K, 0, B.data_ptr(), K, 0, dU.data_ptr(), N,
                                               1.0, None, U.data_ptr(), N, None))
    torch.cuda.synchronize()
    x = U.float().requires_grad_()
    torch.nn.functional.gelu(x).backward(torch.ones_like(x))
    du_ref = (A.float() @ B.float().t()).bfloat16().float() * x.grad
    assert ((dU.float() - du_ref).norm() / du_ref.norm()).item() < 8e-3
    assert tsplit.lib().ts_gemm_bf16_epi(3, M, N, K, A.data_ptr(), K, 0, B.data_ptr(), K, 0, dU.data_ptr(), N, 1.0,
                                         None, U.data_ptr(), N, None) == tsplit.STATUS.index("ERR_ARG")
