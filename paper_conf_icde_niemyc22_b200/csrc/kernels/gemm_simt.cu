// CUDA-core GEMM (FFMA, fp32 accumulate) for fp32 graphs (config 1: "true fp32",
// TF32 would break the 1e-5 tolerance) and for products too small
// or misaligned for the tcgen05/TMA path (e.g. a 2-class classifier).  Same
// strided-operand contract as gemm_tc.
#include "common.cuh"
#include "kernels.h"

namespace tsk {

namespace {
constexpr int TM = 64, TN = 64, TK = 16;

// fp32 inputs accumulate in fp64 (AccT = double): a true-fp32 graph's products are
// then correctly rounded, and a split of the K (sample) dimension changes them only
// by the final fp32 accumulation (split invariance).
template <class TI, class TO, class AccT>
__global__ void __launch_bounds__(256) gemm_simt_kernel(GemmArgs g) {
  __shared__ float As[TK][TM + 4];
  __shared__ float Bs[TK][TN + 4];
  const int bz = blockIdx.z;
  const int b1 = bz % g.nb1, b2 = bz / g.nb1;
  const TI* A = reinterpret_cast<const TI*>(g.a.ptr) + b1 * g.a.bs1 + b2 * g.a.bs2;
  const TI* B = reinterpret_cast<const TI*>(g.b.ptr) + b1 * g.b.bs1 + b2 * g.b.bs2;
  const int m0 = blockIdx.y * TM, n0 = blockIdx.x * TN;
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  AccT acc[4][4] = {};
  for (int k0 = 0; k0 < g.K; k0 += TK) {
    for (int i = threadIdx.x; i < TM * TK; i += 256) {
      int mm, kk;
      if (g.a.mn_major) { mm = i % TM; kk = i / TM; } else { kk = i % TK; mm = i / TK; }
      int m = m0 + mm, k = k0 + kk;
      float v = 0.f;
      if (m < g.M && k < g.K) v = to_f(A[g.a.mn_major ? int64_t(k) * g.a.ld + m : int64_t(m) * g.a.ld + k]);
      As[kk][mm] = v;
    }
    for (int i = threadIdx.x; i < TN * TK; i += 256) {
      int nn, kk;
      if (g.b.mn_major) { nn = i % TN; kk = i / TN; } else { kk = i % TK; nn = i / TK; }
      int n = n0 + nn, k = k0 + kk;
      float v = 0.f;
      if (n < g.N && k < g.K) v = to_f(B[g.b.mn_major ? int64_t(k) * g.b.ld + n : int64_t(n) * g.b.ld + k]);
      Bs[kk][nn] = v;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < TK; ++kk) {
      AccT a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) a[i] = As[kk][ty * 4 + i];
#pragma unroll
      for (int j = 0; j < 4; ++j) b[j] = Bs[kk][tx * 4 + j];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fma(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
  TO* C = reinterpret_cast<TO*>(g.c) + b1 * g.cbs1 + b2 * g.cbs2;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    int m = m0 + ty * 4 + i;
    if (m >= g.M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      int n = n0 + tx * 4 + j;
      if (n >= g.N) continue;
      AccT v = acc[i][j] * AccT(g.alpha);
      if (g.bias)
        v += g.bias_dtype == F32 ? AccT(reinterpret_cast<const float*>(g.bias)[n])
                                 : AccT(to_f(reinterpret_cast<const bf16*>(g.bias)[n]));
      TO* cp = C + int64_t(m) * g.ldc + n;
      if (g.beta != 0.f) v += AccT(g.beta) * AccT(to_f(*cp));
      *cp = from_f<TO>(float(v));
    }
  }
}
// Tiny products (the classifier / pooler of a small batch: M x N of a few thousand outputs,
// K up to thousands): one warp per output, lanes striding K (coalesced for K-major
// operands), a fixed xor-shuffle tree — deterministic, and no 64-step K loop on one CTA.
template <class TI, class TO, class AccT>
__global__ void __launch_bounds__(256) gemm_small_kernel(GemmArgs g) {
  const int64_t w = (int64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t per = int64_t(g.M) * g.N;
  if (w >= per * g.nb1 * g.nb2) return;
  const int bz = int(w / per);
  const int m = int((w % per) / g.N), n = int(w % g.N);
  const int b1 = bz % g.nb1, b2 = bz / g.nb1;
  const TI* A = reinterpret_cast<const TI*>(g.a.ptr) + b1 * g.a.bs1 + b2 * g.a.bs2;
  const TI* B = reinterpret_cast<const TI*>(g.b.ptr) + b1 * g.b.bs1 + b2 * g.b.bs2;
  AccT acc = 0;
  for (int k = lane; k < g.K; k += 32) {
    const float a = to_f(A[g.a.mn_major ? int64_t(k) * g.a.ld + m : int64_t(m) * g.a.ld + k]);
    const float b = to_f(B[g.b.mn_major ? int64_t(k) * g.b.ld + n : int64_t(n) * g.b.ld + k]);
    acc = fma(AccT(a), AccT(b), acc);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if (lane) return;
  TO* cp = reinterpret_cast<TO*>(g.c) + b1 * g.cbs1 + b2 * g.cbs2 + int64_t(m) * g.ldc + n;
  AccT v = acc * AccT(g.alpha);
  if (g.bias)
    v += g.bias_dtype == F32 ? AccT(reinterpret_cast<const float*>(g.bias)[n])
                             : AccT(to_f(reinterpret_cast<const bf16*>(g.bias)[n]));
  if (g.beta != 0.f) v += AccT(g.beta) * AccT(to_f(*cp));
  *cp = from_f<TO>(float(v));
}
}  // namespace

void gemm_simt(const GemmArgs& g, cudaStream_t st) {
  const int64_t outs = int64_t(g.M) * g.N * g.nb1 * g.nb2;
  if (outs <= 16384 && g.K >= 64) {  // tiny output, long reduction: a warp per output
    const int blocks = int((outs * 32 + 255) / 256);
    if (g.in_dtype == F32) {
      if (g.c_dtype == F32) gemm_small_kernel<float, float, double><<<blocks, 256, 0, st>>>(g);
      else gemm_small_kernel<float, bf16, double><<<blocks, 256, 0, st>>>(g);
    } else {
      if (g.c_dtype == F32) gemm_small_kernel<bf16, float, float><<<blocks, 256, 0, st>>>(g);
      else gemm_small_kernel<bf16, bf16, float><<<blocks, 256, 0, st>>>(g);
    }
    return;
  }
  dim3 grid((g.N + TN - 1) / TN, (g.M + TM - 1) / TM, g.nb1 * g.nb2);
  if (g.in_dtype == F32) {
    if (g.c_dtype == F32) gemm_simt_kernel<float, float, double><<<grid, 256, 0, st>>>(g);
    else gemm_simt_kernel<float, bf16, double><<<grid, 256, 0, st>>>(g);
  } else {
    if (g.c_dtype == F32) gemm_simt_kernel<bf16, float, float><<<grid, 256, 0, st>>>(g);
    else gemm_simt_kernel<bf16, bf16, float><<<grid, 256, 0, st>>>(g);
  }
}

}  // namespace tsk
