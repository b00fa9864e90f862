// Staging copies of attribute (height) band splits — DESIGN.md reading D-ATTR, the physical
// merge & split of P:L264 (Fig. 10) for window ops (conv2d, maxpool) whose input or output is
// split along H.
//
//   gather:      S[b, r, w, c] = X[b0 + b, lo + r, w - pad, c]   (rows / columns outside X: fill)
//   scatter-add: dX[b0 + b, h, w, c] += dS[b, h - lo, w + pad, c] for the rows h in [lo, lo+hs) ∩ [0, H)
//
// X is p pieces of hb rows each, piece j = rows [j hb, (j+1) hb) of every sample, stored
// [B, hb, W, C] (an unsplit tensor is one piece of H rows).  Both are HBM-bound copies: one
// 16-byte vector per thread when a pixel row is whole vectors (every activation but the
// 3-channel image), one element otherwise; grid-stride loops over 8 CTAs per SM.
#include "common.cuh"
#include "kernels.h"

namespace tsk {

namespace {

constexpr int kT = 256;

int grid_for(int64_t n) {
  int64_t b = (n + kT - 1) / kT;
  return int(b < 148 * 8 ? b : 148 * 8);
}

template <class T, int V>
__global__ void band_gather_k(BandPieces x, int H, int W, int C, int b0, int nb, int lo, int hs, int pad, T fill,
                              T* __restrict__ out) {
  const int CV = C / V, Wp = W + 2 * pad;
  const int64_t total = int64_t(nb) * hs * Wp * CV;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < total; i += int64_t(gridDim.x) * blockDim.x) {
    const int cv = int(i % CV);
    const int64_t pix = i / CV;
    const int w = int(pix % Wp), r = int((pix / Wp) % hs), b = int(pix / (int64_t(Wp) * hs));
    const int h = lo + r, ww = w - pad;
    T* o = out + pix * C + int64_t(cv) * V;
    if (h >= 0 && h < H && ww >= 0 && ww < W) {
      const int j = h / x.hb;
      const T* src = static_cast<const T*>(x.ptr[j]) + ((int64_t(b0 + b) * x.hb + (h - j * x.hb)) * W + ww) * C +
                     int64_t(cv) * V;
      if constexpr (V * sizeof(T) == 16) {
        *reinterpret_cast<uint4*>(o) = *reinterpret_cast<const uint4*>(src);
      } else {
#pragma unroll
        for (int e = 0; e < V; ++e) o[e] = src[e];
      }
    } else {
#pragma unroll
      for (int e = 0; e < V; ++e) o[e] = fill;
    }
  }
}

template <class T, int V>
__global__ void band_scatter_add_k(const T* __restrict__ src, BandPieces dx, int H, int W, int C, int b0, int nb,
                                   int lo, int hs, int pad, int rlo, int nr) {
  const int CV = C / V, Wp = W + 2 * pad;
  const int64_t total = int64_t(nb) * nr * W * CV;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < total; i += int64_t(gridDim.x) * blockDim.x) {
    const int cv = int(i % CV);
    const int64_t pix = i / CV;
    const int w = int(pix % W), rr = int((pix / W) % nr), b = int(pix / (int64_t(W) * nr));
    const int h = rlo + rr;
    const int j = h / dx.hb;
    T* d = static_cast<T*>(const_cast<void*>(dx.ptr[j])) + ((int64_t(b0 + b) * dx.hb + (h - j * dx.hb)) * W + w) * C +
           int64_t(cv) * V;
    const T* s = src + ((int64_t(b) * hs + (h - lo)) * Wp + w + pad) * C + int64_t(cv) * V;
    if constexpr (V * sizeof(T) == 16) {
      uint4 dv = *reinterpret_cast<const uint4*>(d);
      const uint4 sv = *reinterpret_cast<const uint4*>(s);
      T* dt = reinterpret_cast<T*>(&dv);
      const T* st = reinterpret_cast<const T*>(&sv);
#pragma unroll
      for (int e = 0; e < V; ++e) dt[e] = from_f<T>(to_f(dt[e]) + to_f(st[e]));
      *reinterpret_cast<uint4*>(d) = dv;
    } else {
#pragma unroll
      for (int e = 0; e < V; ++e) d[e] = from_f<T>(to_f(d[e]) + to_f(s[e]));
    }
  }
}

template <class T>
void gather_launch(const BandPieces& x, int H, int W, int C, int b0, int nb, int lo, int hs, int pad, T fill, void* out,
                   cudaStream_t st) {
  constexpr int V = 16 / sizeof(T);
  const int64_t pix = int64_t(nb) * hs * (W + 2 * pad);
  if (C % V == 0)
    band_gather_k<T, V><<<grid_for(pix * (C / V)), kT, 0, st>>>(x, H, W, C, b0, nb, lo, hs, pad, fill,
                                                                  static_cast<T*>(out));
  else
    band_gather_k<T, 1><<<grid_for(pix * C), kT, 0, st>>>(x, H, W, C, b0, nb, lo, hs, pad, fill, static_cast<T*>(out));
}

template <class T>
void scatter_launch(const void* src, const BandPieces& dx, int H, int W, int C, int b0, int nb, int lo, int hs, int pad,
                    cudaStream_t st) {
  constexpr int V = 16 / sizeof(T);
  const int rlo = lo > 0 ? lo : 0, rhi = lo + hs - 1 < H - 1 ? lo + hs - 1 : H - 1;
  const int nr = rhi - rlo + 1;
  if (nr <= 0) return;
  const int64_t pix = int64_t(nb) * nr * W;
  if (C % V == 0)
    band_scatter_add_k<T, V><<<grid_for(pix * (C / V)), kT, 0, st>>>(static_cast<const T*>(src), dx, H, W, C, b0, nb,
                                                                       lo, hs, pad, rlo, nr);
  else
    band_scatter_add_k<T, 1><<<grid_for(pix * C), kT, 0, st>>>(static_cast<const T*>(src), dx, H, W, C, b0, nb, lo, hs,
                                                                 pad, rlo, nr);
}

}  // namespace

void band_gather(int dt, const BandPieces& x, int H, int W, int C, int b0, int nb, int lo, int hs, int pad,
                 int neg_inf_fill, void* out, cudaStream_t st) {
  if (dt == BF16)
    gather_launch<bf16>(x, H, W, C, b0, nb, lo, hs, pad, neg_inf_fill ? __float2bfloat16_rn(-INFINITY) : bf16(0.f), out,
                        st);
  else
    gather_launch<float>(x, H, W, C, b0, nb, lo, hs, pad, neg_inf_fill ? -INFINITY : 0.f, out, st);
}

void band_scatter_add(int dt, const void* src, const BandPieces& dx, int H, int W, int C, int b0, int nb, int lo, int hs,
                      int pad, cudaStream_t st) {
  if (dt == BF16) scatter_launch<bf16>(src, dx, H, W, C, b0, nb, lo, hs, pad, st);
  else scatter_launch<float>(src, dx, H, W, C, b0, nb, lo, hs, pad, st);
}

}  // namespace tsk
