// Staging copies of attribute (height / width) band splits — DESIGN.md reading D-ATTR, the
// physical merge & split of P:L264 (Fig. 10) for window ops (conv2d, maxpool) whose input or
// output is split along H or W.
//
//   gather:      S[b, r, c', ch] = X[b0 + b, rlo + r, clo + c', ch]   (outside X: fill)
//   scatter-add: dX[b0 + b, h, w, ch] += dS[b, h - rlo, w - clo, ch] for (h, w) in the rectangle ∩ X
//
// X is p pieces of hb rows (piece j = rows [j hb, (j+1) hb) of every sample, stored
// [B, hb, W, C]) or of hb columns ([B, H, hb, C]); an unsplit tensor is one piece of H rows.
// Both are HBM-bound copies: one 16-byte vector per thread when a pixel row is whole vectors (every activation but the
// 3-channel image), one element otherwise; one staged row per blockIdx.y, ~8 CTAs per SM.
#include "common.cuh"
#include "kernels.h"

namespace tsk {

namespace {

constexpr int kT = 256;

// element offset of (b, h, w, c) inside its piece, and the piece (axis 3: channel blocks of
// hb channels, D-CH's staged merge); 32-bit index math (a staged rectangle holds < 2^31 vectors)
__device__ __forceinline__ int64_t band_off(const BandPieces& x, int H, int W, int C, int b, int h, int w, int c,
                                            int& j) {
  if (x.axis == 1) {
    j = h / x.hb;
    return ((int64_t(b) * x.hb + (h - j * x.hb)) * W + w) * C + c;
  }
  if (x.axis == 2) {
    j = w / x.hb;
    return ((int64_t(b) * H + h) * x.hb + (w - j * x.hb)) * C + c;
  }
  j = c / x.hb;
  return ((int64_t(b) * H + h) * W + w) * x.hb + (c - j * x.hb);
}

// one staged row (sample b, row r) per blockIdx.y (grid-stride over rows), its ws * C / V
// vectors over the x dimension: the row's range check and base offsets are per block
template <class T, int V>
__global__ void band_gather_k(BandPieces x, int H, int W, int C, Rect r, T fill, T* __restrict__ out) {
  const int CV = C / V, nv = r.ws * CV, nrows = r.nb * r.hs;
  for (int row = blockIdx.y; row < nrows; row += gridDim.y) {
    const int b = row / r.hs, h = r.rlo + (row - b * r.hs);
    T* orow = out + int64_t(row) * r.ws * C;
    const bool hin = h >= 0 && h < H;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nv; i += gridDim.x * blockDim.x) {
      const int w = i / CV, cv = i - w * CV;
      const int ww = r.clo + w;
      T* o = orow + int64_t(w) * C + cv * V;
      if (hin && ww >= 0 && ww < W) {
        int j;
        const int64_t off = band_off(x, H, W, C, r.b0 + b, h, ww, cv * V, j);
        const T* src = static_cast<const T*>(x.ptr[j]) + off;
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
}

// over the rectangle's pixels inside X: rows [h0, h0 + nh) x columns [w0, w0 + nw), one
// (sample, row) per blockIdx.y
template <class T, int V>
__global__ void band_scatter_add_k(const T* __restrict__ src, BandPieces dx, int H, int W, int C, Rect r, int h0,
                                   int nh, int w0, int nw) {
  const int CV = C / V, nv = nw * CV, nrows = r.nb * nh;
  for (int row = blockIdx.y; row < nrows; row += gridDim.y) {
    const int b = row / nh, h = h0 + (row - b * nh);
    const T* srow = src + (int64_t(b) * r.hs + (h - r.rlo)) * r.ws * C;
    for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < nv; i += gridDim.x * blockDim.x) {
      const int wi = i / CV, cv = i - wi * CV;
      const int w = w0 + wi;
      int j;
      const int64_t off = band_off(dx, H, W, C, r.b0 + b, h, w, cv * V, j);
      T* d = static_cast<T*>(const_cast<void*>(dx.ptr[j])) + off;
      const T* s = srow + int64_t(w - r.clo) * C + cv * V;
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
}

// (x blocks per row, rows in flight): about 8 CTAs of 256 threads per SM in all
dim3 grid2(int nv, int nrows) {
  const int bx = (nv + kT - 1) / kT;
  int by = (148 * 8) / bx;
  by = by < 1 ? 1 : by;
  by = by < nrows ? by : nrows;
  by = by < 65535 ? by : 65535;
  return dim3(unsigned(bx), unsigned(by));
}

template <class T>
void gather_launch(const BandPieces& x, int H, int W, int C, const Rect& r, T fill, void* out, cudaStream_t st) {
  constexpr int V = 16 / sizeof(T);
  if (C % V == 0 && (x.axis != 3 || x.hb % V == 0))  // (a vector never straddles two channel blocks)
    band_gather_k<T, V><<<grid2(r.ws * (C / V), r.nb * r.hs), kT, 0, st>>>(x, H, W, C, r, fill, static_cast<T*>(out));
  else
    band_gather_k<T, 1><<<grid2(r.ws * C, r.nb * r.hs), kT, 0, st>>>(x, H, W, C, r, fill, static_cast<T*>(out));
}

template <class T>
void scatter_launch(const void* src, const BandPieces& dx, int H, int W, int C, const Rect& r, cudaStream_t st) {
  constexpr int V = 16 / sizeof(T);
  const int h0 = r.rlo > 0 ? r.rlo : 0, h1 = r.rlo + r.hs < H ? r.rlo + r.hs : H;
  const int w0 = r.clo > 0 ? r.clo : 0, w1 = r.clo + r.ws < W ? r.clo + r.ws : W;
  if (h1 <= h0 || w1 <= w0) return;
  const int nrows = r.nb * (h1 - h0);
  if (C % V == 0 && (dx.axis != 3 || dx.hb % V == 0))
    band_scatter_add_k<T, V><<<grid2((w1 - w0) * (C / V), nrows), kT, 0, st>>>(static_cast<const T*>(src), dx, H, W,
                                                                                 C, r, h0, h1 - h0, w0, w1 - w0);
  else
    band_scatter_add_k<T, 1><<<grid2((w1 - w0) * C, nrows), kT, 0, st>>>(static_cast<const T*>(src), dx, H, W, C, r,
                                                                           h0, h1 - h0, w0, w1 - w0);
}

}  // namespace

void band_gather(int dt, const BandPieces& x, int H, int W, int C, const Rect& r, int neg_inf_fill, void* out,
                 cudaStream_t st) {
  if (dt == BF16)
    gather_launch<bf16>(x, H, W, C, r, neg_inf_fill ? __float2bfloat16_rn(-INFINITY) : bf16(0.f), out, st);
  else
    gather_launch<float>(x, H, W, C, r, neg_inf_fill ? -INFINITY : 0.f, out, st);
}

void band_scatter_add(int dt, const void* src, const BandPieces& dx, int H, int W, int C, const Rect& r,
                      cudaStream_t st) {
  if (dt == BF16) scatter_launch<bf16>(src, dx, H, W, C, r, st);
  else scatter_launch<float>(src, dx, H, W, C, r, st);
}

}  // namespace tsk
