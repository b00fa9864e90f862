// Direct CUDA-core convolution for the image layer (C <= 4 input channels: VGG-16 conv0,
// ResNet-50 stem) — the conv micro-op of SURVEY.md §8(a) a6/a8 where the implicit GEMM's
// reduction (R*S*C = 27 or 147) is too short and too ragged for tcgen05 tiles: the gather
// kernel spends its time assembling 3-channel rows, while here the input patch sits in
// shared memory (fp32) and every weight / pixel value is reused from registers.
//   fprop  y[n,p,q,k] = sum_{r,s,c} x[n, p*st-pad+r, q*st-pad+s, c] w[k,r,s,c] + bias[k]
//          block = one output row segment of 32 pixels x 64 channels; thread = 8
//          consecutive pixels of one channel, so for a fixed (r, c) the 8 + (S-1)*... input
//          values of a row stay in registers across the S taps.
//   wgrad  dw[k,r,s,c] (+)= sum over the micro-op's pixels of dy[n,p,q,k] x[...]:
//          block = a band of output rows of one image; thread = one channel k and a quarter
//          of the (r,s,c) taps; per-block partials are added with fp32 red.add (the split-K
//          merge of the tcgen05 wgrad, P:L260 merge-by-sum).
// dgrad is never needed for the image layer (the input takes no gradient).
#include <cstdint>

#include "common.cuh"
#include "kernels.h"

namespace tsk {

namespace {

constexpr int kTQ = 32;       // output pixels per fprop block
constexpr int kPX = 8;        // pixels per thread (fprop)
constexpr int kMaxRSC = 196;  // 7 x 7 x 4

__global__ void __launch_bounds__(256) conv_direct_fprop(const bf16* __restrict__ x, const bf16* __restrict__ w,
                                                         const bf16* __restrict__ bias, bf16* __restrict__ y,
                                                         int H, int W, int C, int K, int R, int S, int P, int Q,
                                                         int st, int pad) {
  extern __shared__ float sm[];
  const int RSC = R * S * C;
  const int cols = (kTQ - 1) * st + S;  // input columns of the segment
  float* wt = sm;                        // [RSC][64] (this block's 64 output channels)
  float* xs = sm + RSC * 64;             // [R][cols][C]
  const int q0 = blockIdx.x * kTQ, p = blockIdx.y, n = blockIdx.z / (K / 64), kb = blockIdx.z % (K / 64);
  const int tid = threadIdx.x;
  for (int i = tid; i < RSC * 64; i += 256) {
    const int k = i & 63, rsc = i >> 6;
    wt[i] = to_f(w[int64_t(kb * 64 + k) * RSC + rsc]);
  }
  const int h0 = p * st - pad, w0 = q0 * st - pad;
  for (int i = tid; i < R * cols * C; i += 256) {
    const int c = i % C, col = (i / C) % cols, r = i / (C * cols);
    const int hh = h0 + r, ww = w0 + col;
    xs[i] = (hh >= 0 && hh < H && ww >= 0 && ww < W) ? to_f(x[((int64_t(n) * H + hh) * W + ww) * C + c]) : 0.f;
  }
  __syncthreads();
  const int k = tid & 63, g = tid >> 6;  // channel, group of kPX consecutive pixels
  float acc[kPX];
  const float b = bias ? to_f(bias[kb * 64 + k]) : 0.f;
#pragma unroll
  for (int j = 0; j < kPX; ++j) acc[j] = b;
  const int qs = g * kPX;  // first pixel of this thread within the segment
  for (int r = 0; r < R; ++r)
    for (int c = 0; c < C; ++c) {
      const float* xrow = xs + (r * cols) * C + c;
      for (int s = 0; s < S; ++s) {
        const float wv = wt[((r * S + s) * C + c) * 64 + k];
#pragma unroll
        for (int j = 0; j < kPX; ++j) acc[j] = fmaf(wv, xrow[((qs + j) * st + s) * C], acc[j]);
      }
    }
#pragma unroll
  for (int j = 0; j < kPX; ++j) {
    const int q = q0 + qs + j;
    if (q < Q) y[((int64_t(n) * P + p) * Q + q) * K + kb * 64 + k] = from_f<bf16>(acc[j]);
  }
}

constexpr int kWRows = 4;  // output rows per wgrad block

template <int NT>  // taps per thread: ceil(R S C / 4), compile-time so the accumulators stay in registers
__global__ void __launch_bounds__(256) conv_direct_wgrad(const bf16* __restrict__ x, const bf16* __restrict__ dy,
                                                         float* __restrict__ dw, int H, int W, int C, int K, int R,
                                                         int S, int P, int Q, int st, int pad) {
  extern __shared__ float sm[];
  const int RSC = R * S * C;
  const int rows_in = (kWRows - 1) * st + R;
  float* xs = sm;  // [rows_in][W + 2 pad][C]
  const int Wp = W + 2 * pad;
  const int pb = blockIdx.x, n = blockIdx.y, kb = blockIdx.z;
  const int p0 = pb * kWRows;
  const int tid = threadIdx.x;
  const int h0 = p0 * st - pad;
  for (int i = tid; i < rows_in * Wp * C; i += 256) {
    const int c = i % C, col = (i / C) % Wp, r = i / (C * Wp);
    const int hh = h0 + r, ww = col - pad;
    xs[i] = (hh >= 0 && hh < H && ww >= 0 && ww < W) ? to_f(x[((int64_t(n) * H + hh) * W + ww) * C + c]) : 0.f;
  }
  __syncthreads();
  const int k = tid & 63, g = tid >> 6;
  // this thread's taps: rsc = g, g + 4, g + 8, ... (a tap past R S C reads offset 0, unused)
  float acc[NT];
  int off[NT];
#pragma unroll
  for (int i = 0; i < NT; ++i) {
    const int rsc = g + 4 * i;
    const int c = rsc % C, s = (rsc / C) % S, r = rsc / (C * S);
    off[i] = rsc < RSC ? (r * Wp + s) * C + c : 0;
    acc[i] = 0.f;
  }
  const int prows = min(kWRows, P - p0);
  for (int pp = 0; pp < prows; ++pp) {
    const bf16* dyr = dy + ((int64_t(n) * P + p0 + pp) * Q) * K + kb * 64 + k;
    const float* xr = xs + (pp * st) * Wp * C;
    for (int q = 0; q < Q; ++q) {
      const float d = to_f(dyr[int64_t(q) * K]);
      const float* xq = xr + (q * st) * C;
#pragma unroll
      for (int i = 0; i < NT; ++i) acc[i] = fmaf(d, xq[off[i]], acc[i]);
    }
  }
#pragma unroll
  for (int i = 0; i < NT; ++i)
    if (g + 4 * i < RSC) atomicAdd(dw + int64_t(kb * 64 + k) * RSC + g + 4 * i, acc[i]);
}

}  // namespace

bool conv_direct(int mode, const ConvArgs& a, void* out, const void* bias, int acc, cudaStream_t st) {
  if (a.dtype != BF16 || a.C > 4 || a.K % 64 || a.R * a.S * a.C > kMaxRSC || mode == 2) return false;
  const int RSC = a.R * a.S * a.C;
  if (mode == 1) {
    const int cols = (kTQ - 1) * a.stride + a.S;
    const size_t smem = (size_t(RSC) * 64 + size_t(a.R) * cols * a.C) * 4;
    if (smem > 200 * 1024) return false;
    static bool attr = false;
    if (!attr) {
      cudaFuncSetAttribute(conv_direct_fprop, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
      attr = true;
    }
    dim3 grid((a.Q + kTQ - 1) / kTQ, a.P, a.n * (a.K / 64));
    conv_direct_fprop<<<grid, 256, smem, st>>>(static_cast<const bf16*>(a.x), static_cast<const bf16*>(a.w),
                                               static_cast<const bf16*>(bias), static_cast<bf16*>(out), a.H, a.W,
                                               a.C, a.K, a.R, a.S, a.P, a.Q, a.stride, a.pad);
    return true;
  }
  const int rows_in = (kWRows - 1) * a.stride + a.R;
  const size_t smem = size_t(rows_in) * (a.W + 2 * a.pad) * a.C * 4;
  if (smem > 200 * 1024) return false;
  float* dw = static_cast<float*>(out);
  const int64_t nw = int64_t(a.K) * RSC;
  if (!acc) cudaMemsetAsync(dw, 0, size_t(nw) * 4, st);
  dim3 grid((a.P + kWRows - 1) / kWRows, a.n, a.K / 64);
  auto go = [&](auto kern) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    kern<<<grid, 256, smem, st>>>(static_cast<const bf16*>(a.x), static_cast<const bf16*>(a.dy), dw, a.H, a.W, a.C,
                                  a.K, a.R, a.S, a.P, a.Q, a.stride, a.pad);
  };
  const int nt = (RSC + 3) / 4;
  if (nt <= 7) go(conv_direct_wgrad<7>);
  else if (nt <= 16) go(conv_direct_wgrad<16>);
  else if (nt <= 37) go(conv_direct_wgrad<37>);
  else go(conv_direct_wgrad<49>);
  return true;
}

}  // namespace tsk
