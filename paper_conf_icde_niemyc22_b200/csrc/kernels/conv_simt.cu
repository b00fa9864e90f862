// Direct convolution on CUDA cores for fp32 graphs (true fp32 with fp64
// accumulation: split changes only the final fp32 accumulation) and
// for shapes the tcgen05 implicit GEMM does not take.  Same index maps as
// conv_tc.cu (fprop / dgrad / wgrad, NHWC x KRSC).
#include "common.cuh"
#include "kernels.h"

namespace tsk {

namespace {

template <class T, class AccT>
__global__ void conv_fprop_simt(ConvArgs a, T* y, const T* bias) {
  const T* x = static_cast<const T*>(a.x);
  const T* w = static_cast<const T*>(a.w);
  const int64_t total = int64_t(a.n) * a.P * a.Q * a.K;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < total; i += int64_t(gridDim.x) * blockDim.x) {
    const int ko = int(i % a.K);
    const int64_t m = i / a.K;
    const int q = int(m % a.Q), p = int((m / a.Q) % a.P), n = int(m / (int64_t(a.Q) * a.P));
    AccT s = 0;
    for (int r = 0; r < a.R; ++r) {
      const int ih = p * a.stride - a.pad + r;
      if (ih < 0 || ih >= a.H) continue;
      for (int t = 0; t < a.S; ++t) {
        const int iw = q * a.stride - a.pad + t;
        if (iw < 0 || iw >= a.W) continue;
        const T* xp = x + ((int64_t(n) * a.H + ih) * a.W + iw) * a.C;
        const T* wp = w + ((int64_t(ko) * a.R + r) * a.S + t) * a.C;
        for (int c = 0; c < a.C; ++c) s += AccT(to_f(xp[c])) * AccT(to_f(wp[c]));
      }
    }
    if (bias) s += AccT(to_f(bias[ko]));
    y[i] = from_f<T>(float(s));
  }
}

template <class T, class AccT>
__global__ void conv_dgrad_simt(ConvArgs a, T* dx, int acc) {
  const T* dy = static_cast<const T*>(a.dy);
  const T* w = static_cast<const T*>(a.w);
  const int64_t total = int64_t(a.n) * a.H * a.W * a.C;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < total; i += int64_t(gridDim.x) * blockDim.x) {
    const int c = int(i % a.C);
    const int64_t m = i / a.C;
    const int wq = int(m % a.W), h = int((m / a.W) % a.H), n = int(m / (int64_t(a.W) * a.H));
    AccT s = 0;
    for (int r = 0; r < a.R; ++r) {
      const int ph = h + a.pad - r;
      if (ph < 0 || ph % a.stride) continue;
      const int p = ph / a.stride;
      if (p >= a.P) continue;
      for (int t = 0; t < a.S; ++t) {
        const int pw = wq + a.pad - t;
        if (pw < 0 || pw % a.stride) continue;
        const int q = pw / a.stride;
        if (q >= a.Q) continue;
        const T* dyp = dy + ((int64_t(n) * a.P + p) * a.Q + q) * a.K;
        for (int ko = 0; ko < a.K; ++ko)
          s += AccT(to_f(dyp[ko])) * AccT(to_f(w[((int64_t(ko) * a.R + r) * a.S + t) * a.C + c]));
      }
    }
    float v = float(s);
    if (acc) v += to_f(dx[i]);
    dx[i] = from_f<T>(v);
  }
}

template <class T, class AccT>
__global__ void conv_wgrad_simt(ConvArgs a, float* dw, int acc) {
  const T* x = static_cast<const T*>(a.x);
  const T* dy = static_cast<const T*>(a.dy);
  const int64_t total = int64_t(a.K) * a.R * a.S * a.C;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < total; i += int64_t(gridDim.x) * blockDim.x) {
    const int c = int(i % a.C);
    const int t = int((i / a.C) % a.S), r = int((i / (int64_t(a.C) * a.S)) % a.R);
    const int ko = int(i / (int64_t(a.C) * a.S * a.R));
    AccT s = 0;
    for (int n = 0; n < a.n; ++n)
      for (int p = 0; p < a.P; ++p) {
        const int ih = p * a.stride - a.pad + r;
        if (ih < 0 || ih >= a.H) continue;
        for (int q = 0; q < a.Q; ++q) {
          const int iw = q * a.stride - a.pad + t;
          if (iw < 0 || iw >= a.W) continue;
          s += AccT(to_f(x[((int64_t(n) * a.H + ih) * a.W + iw) * a.C + c])) *
               AccT(to_f(dy[((int64_t(n) * a.P + p) * a.Q + q) * a.K + ko]));
        }
      }
    dw[i] = float(s) + (acc ? dw[i] : 0.f);
  }
}

int grid_for(int64_t total) {
  int64_t b = (total + 255) / 256;
  return int(b < 148 * 16 ? b : 148 * 16);
}

}  // namespace

void conv_simt(int mode, const ConvArgs& a, void* out, const void* bias, int acc, cudaStream_t st) {
  const bool f32 = a.dtype == F32;
  if (mode == 1) {
    const int g = grid_for(int64_t(a.n) * a.P * a.Q * a.K);
    if (f32) conv_fprop_simt<float, double><<<g, 256, 0, st>>>(a, static_cast<float*>(out), static_cast<const float*>(bias));
    else conv_fprop_simt<bf16, float><<<g, 256, 0, st>>>(a, static_cast<bf16*>(out), static_cast<const bf16*>(bias));
  } else if (mode == 2) {
    const int g = grid_for(int64_t(a.n) * a.H * a.W * a.C);
    if (f32) conv_dgrad_simt<float, double><<<g, 256, 0, st>>>(a, static_cast<float*>(out), acc);
    else conv_dgrad_simt<bf16, float><<<g, 256, 0, st>>>(a, static_cast<bf16*>(out), acc);
  } else {
    const int g = grid_for(int64_t(a.K) * a.R * a.S * a.C);
    if (f32) conv_wgrad_simt<float, double><<<g, 256, 0, st>>>(a, static_cast<float*>(out), acc);
    else conv_wgrad_simt<bf16, float><<<g, 256, 0, st>>>(a, static_cast<float*>(out), acc);
  }
}

}  // namespace tsk
