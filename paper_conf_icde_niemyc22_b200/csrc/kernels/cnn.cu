// CNN micro-op kernels: train-mode batch normalisation whose statistics span the
// whole batch even when the tensor is split ("merge ...
// required by ... batch normalization"), max/avg pooling.  NHWC: a row is one
// pixel's C channels, so every kernel moves 16-byte channel vectors (HBM-bound,
// coalesced) and a sample split is a row range.
//
// BN statistics are two-phase and deterministic: each block reduces a fixed row
// range of one piece to per-channel fp32 partial sums (shifted by the first row to
// avoid cancellation), then one kernel adds the partials in fp64 in block order.
#include "common.cuh"
#include "kernels.h"

namespace tsk {

namespace {

constexpr int kT = 256;
constexpr uint64_t kTicketBytes = 4096;  // tail of the workspace used by column_sum

template <class T>
struct VecT {
  static constexpr int N = 16 / sizeof(T);
};
template <class T>
__device__ __forceinline__ void ldv(const T* p, float* v) {
  uint4 u = *reinterpret_cast<const uint4*>(p);
  const T* t = reinterpret_cast<const T*>(&u);
#pragma unroll
  for (int i = 0; i < VecT<T>::N; ++i) v[i] = to_f(t[i]);
}
template <class T>
__device__ __forceinline__ void stv(T* p, const float* v) {
  uint4 u;
  T* t = reinterpret_cast<T*>(&u);
#pragma unroll
  for (int i = 0; i < VecT<T>::N; ++i) t[i] = from_f<T>(v[i]);
  *reinterpret_cast<uint4*>(p) = u;
}

// Segments: the finer of the piece lists cuts the batch into `nseg` equal row
// ranges; `gps` blocks share one segment.  Row r of segment sg in list L lives in
// piece sg / (nseg / L.np) at local row (sg % (nseg / L.np)) * seg_rows + r.
__device__ __forceinline__ const uint8_t* seg_ptr(const PieceList& L, int nseg, int sg, int64_t seg_rows,
                                                  int64_t row_bytes) {
  const int per = nseg / L.np;
  return static_cast<const uint8_t*>(L.ptr[sg / per]) + int64_t(sg % per) * seg_rows * row_bytes;
}

// fp32 graphs accumulate in fp64 (like gemm_simt: a split then changes a sum by at
// most the final fp32 rounding); bf16 graphs in fp32.
template <class T>
struct AccOf {
  typedef float type;
};
template <>
struct AccOf<float> {
  typedef double type;
};

// mode 0: sums of (x - shift), (x - shift)^2.  mode 1: sums of dy, dy * xhat.
template <class T, int MODE>
__global__ void __launch_bounds__(kT) bn_partials(PieceList a, PieceList b, int C, int nseg, int gps,
                                                  int64_t seg_rows, const float* stats,
                                                  typename AccOf<T>::type* ws) {
  typedef typename AccOf<T>::type Acc;
  constexpr int V = VecT<T>::N;
  __shared__ Acc sh0[kT * V], sh1[kT * V];
  const int VPR = C / V;
  const int rpi = kT / VPR;  // rows in flight per block iteration
  const int t = threadIdx.x;
  const int cv = t % VPR, roff = t / VPR;
  const int sg = blockIdx.x / gps, sub = blockIdx.x % gps;
  const int64_t r0 = seg_rows * sub / gps, r1 = seg_rows * (sub + 1) / gps;
  const int64_t rb = int64_t(C) * sizeof(T);
  const T* pa = reinterpret_cast<const T*>(seg_ptr(a, nseg, sg, seg_rows, rb));
  const T* pb = MODE == 1 ? reinterpret_cast<const T*>(seg_ptr(b, nseg, sg, seg_rows, rb)) : nullptr;
  Acc s0[V] = {}, s1[V] = {};
  float sh[V], mu[V], rs[V];
  if (roff < rpi) {
    if (MODE == 0) {
      ldv(static_cast<const T*>(a.ptr[0]) + cv * V, sh);  // shift = first row of the batch
    } else {
#pragma unroll
      for (int i = 0; i < V; ++i) {
        mu[i] = stats[cv * V + i];
        rs[i] = stats[C + cv * V + i];
      }
    }
    for (int64_t r = r0 + roff; r < r1; r += rpi) {
      float x[V];
      ldv(pa + r * C + cv * V, x);
      if (MODE == 0) {
#pragma unroll
        for (int i = 0; i < V; ++i) {
          const Acc d = Acc(x[i]) - Acc(sh[i]);
          s0[i] += d;
          s1[i] += d * d;
        }
      } else {
        float xv[V];
        ldv(pb + r * C + cv * V, xv);
#pragma unroll
        for (int i = 0; i < V; ++i) {
          s0[i] += x[i];
          s1[i] += Acc(x[i]) * ((Acc(xv[i]) - Acc(mu[i])) * Acc(rs[i]));
        }
      }
    }
  }
#pragma unroll
  for (int i = 0; i < V; ++i) {
    sh0[t * V + i] = s0[i];
    sh1[t * V + i] = s1[i];
  }
  __syncthreads();
  // channel c = cv*V + i was accumulated by threads roff*VPR + cv
  for (int c = t; c < C; c += kT) {
    const int cvv = c / V, i = c % V;
    Acc u0 = 0, u1 = 0;
    for (int ro = 0; ro < rpi; ++ro) {
      u0 += sh0[(ro * VPR + cvv) * V + i];
      u1 += sh1[(ro * VPR + cvv) * V + i];
    }
    ws[int64_t(blockIdx.x) * 2 * C + c] = u0;
    ws[int64_t(blockIdx.x) * 2 * C + C + c] = u1;
  }
}

template <class T>
__global__ void bn_finish_stats(const typename AccOf<T>::type* ws, int G, int C, int64_t m, float eps, const T* shift, float* stats) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= C) return;
  double s = 0, q = 0;
  for (int g = 0; g < G; ++g) {
    s += ws[int64_t(g) * 2 * C + c];
    q += ws[int64_t(g) * 2 * C + C + c];
  }
  const double ms = s / double(m);
  double var = q / double(m) - ms * ms;
  if (var < 0) var = 0;
  stats[c] = float(double(to_f(shift[c])) + ms);
  stats[C + c] = float(1.0 / sqrt(var + double(eps)));
}

template <class T>
__global__ void bn_finish_bwd(const typename AccOf<T>::type* ws, int G, int C, const T* gamma, float* stats, float* dgamma,
                              float* dbeta, int pacc) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= C) return;
  double s = 0, q = 0;
  for (int g = 0; g < G; ++g) {
    s += ws[int64_t(g) * 2 * C + c];
    q += ws[int64_t(g) * 2 * C + C + c];
  }
  const double gm = to_f(gamma[c]);
  stats[2 * C + c] = float(gm * s);
  stats[3 * C + c] = float(gm * q);
  dbeta[c] = float(s) + (pacc ? dbeta[c] : 0.f);
  dgamma[c] = float(q) + (pacc ? dgamma[c] : 0.f);
}

template <class T>
__global__ void bn_apply_k(const T* __restrict__ x, const float* __restrict__ stats, const T* __restrict__ g,
                           const T* __restrict__ b, T* __restrict__ y, int64_t nv, int C) {
  constexpr int V = VecT<T>::N;
  for (int64_t v = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; v < nv; v += int64_t(gridDim.x) * blockDim.x) {
    const int c0 = int((v * V) % C);
    float xv[V], o[V];
    ldv(x + v * V, xv);
#pragma unroll
    for (int i = 0; i < V; ++i) {
      const int c = c0 + i;
      o[i] = (xv[i] - stats[c]) * stats[C + c] * to_f(g[c]) + to_f(b[c]);
    }
    stv(y + v * V, o);
  }
}

template <class T>
__global__ void bn_bwd_apply_k(const T* __restrict__ dy, const T* __restrict__ x, const float* __restrict__ stats,
                               const T* __restrict__ g, T* dx, int acc, int64_t nv, int C, float inv_m) {
  constexpr int V = VecT<T>::N;
  for (int64_t v = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; v < nv; v += int64_t(gridDim.x) * blockDim.x) {
    const int c0 = int((v * V) % C);
    float d[V], xv[V], o[V];
    ldv(dy + v * V, d);
    ldv(x + v * V, xv);
    if (acc) ldv(dx + v * V, o);
#pragma unroll
    for (int i = 0; i < V; ++i) {
      const int c = c0 + i;
      const float rs = stats[C + c];
      const float xh = (xv[i] - stats[c]) * rs;
      const float r = rs * (d[i] * to_f(g[c]) - stats[2 * C + c] * inv_m - xh * stats[3 * C + c] * inv_m);
      o[i] = acc ? o[i] + r : r;
    }
    stv(dx + v * V, o);
  }
}

// ------------------------------------------------------------------ pooling
template <class T>
__global__ void maxpool_fwd_k(const T* __restrict__ x, T* __restrict__ y, int n, int H, int W, int C, int P, int Q,
                              int k, int st, int pad) {
  constexpr int V = VecT<T>::N;
  const int CV = C / V;
  const int64_t total = int64_t(n) * P * Q * CV;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < total; i += int64_t(gridDim.x) * blockDim.x) {
    const int cv = int(i % CV);
    const int64_t pix = i / CV;
    const int q = int(pix % Q), p = int((pix / Q) % P), nn = int(pix / (int64_t(P) * Q));
    float m[V];
#pragma unroll
    for (int e = 0; e < V; ++e) m[e] = -INFINITY;
    for (int r = 0; r < k; ++r) {
      const int ih = p * st - pad + r;
      if (ih < 0 || ih >= H) continue;
      for (int s = 0; s < k; ++s) {
        const int iw = q * st - pad + s;
        if (iw < 0 || iw >= W) continue;
        float xv[V];
        ldv(x + ((int64_t(nn) * H + ih) * W + iw) * C + cv * V, xv);
#pragma unroll
        for (int e = 0; e < V; ++e) m[e] = fmaxf(m[e], xv[e]);
      }
    }
    stv(y + pix * C + cv * V, m);
  }
}

// input-centric: dx[h,w] = sum over the windows whose first maximum (row-major) is (h,w)
template <class T>
__global__ void maxpool_bwd_k(const T* __restrict__ dy, const T* __restrict__ x, T* dx, int acc, int n, int H, int W,
                              int C, int P, int Q, int k, int st, int pad) {
  constexpr int V = VecT<T>::N;
  const int CV = C / V;
  const int64_t total = int64_t(n) * H * W * CV;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < total; i += int64_t(gridDim.x) * blockDim.x) {
    const int cv = int(i % CV);
    const int64_t pix = i / CV;
    const int w = int(pix % W), h = int((pix / W) % H), nn = int(pix / (int64_t(H) * W));
    float g[V] = {};
    // windows p with p*st - pad <= h <= p*st - pad + k - 1
    int plo = h + pad - k + 1;
    plo = plo <= 0 ? 0 : (plo + st - 1) / st;
    const int phi = min(P - 1, (h + pad) / st);
    int qlo = w + pad - k + 1;
    qlo = qlo <= 0 ? 0 : (qlo + st - 1) / st;
    const int qhi = min(Q - 1, (w + pad) / st);
    for (int p = plo; p <= phi; ++p)
      for (int q = qlo; q <= qhi; ++q) {
        float m[V];
        int arg[V];
#pragma unroll
        for (int e = 0; e < V; ++e) {
          m[e] = -INFINITY;
          arg[e] = -1;
        }
        for (int r = 0; r < k; ++r) {
          const int ih = p * st - pad + r;
          if (ih < 0 || ih >= H) continue;
          for (int s = 0; s < k; ++s) {
            const int iw = q * st - pad + s;
            if (iw < 0 || iw >= W) continue;
            float xv[V];
            ldv(x + ((int64_t(nn) * H + ih) * W + iw) * C + cv * V, xv);
#pragma unroll
            for (int e = 0; e < V; ++e)
              if (xv[e] > m[e]) {
                m[e] = xv[e];
                arg[e] = ih * W + iw;
              }
          }
        }
        float d[V];
        ldv(dy + ((int64_t(nn) * P + p) * Q + q) * C + cv * V, d);
#pragma unroll
        for (int e = 0; e < V; ++e)
          if (arg[e] == h * W + w) g[e] += d[e];
      }
    if (acc) {
      float o[V];
      ldv(dx + pix * C + cv * V, o);
#pragma unroll
      for (int e = 0; e < V; ++e) g[e] += o[e];
    }
    stv(dx + pix * C + cv * V, g);
  }
}

template <class T>
__global__ void avgpool_fwd_k(const T* __restrict__ x, T* __restrict__ y, int n, int HW, int C) {
  constexpr int V = VecT<T>::N;
  const int CV = C / V;
  const int64_t total = int64_t(n) * CV;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < total; i += int64_t(gridDim.x) * blockDim.x) {
    const int cv = int(i % CV), nn = int(i / CV);
    float s[V] = {};
    for (int j = 0; j < HW; ++j) {
      float xv[V];
      ldv(x + (int64_t(nn) * HW + j) * C + cv * V, xv);
#pragma unroll
      for (int e = 0; e < V; ++e) s[e] += xv[e];
    }
#pragma unroll
    for (int e = 0; e < V; ++e) s[e] /= float(HW);
    stv(y + int64_t(nn) * C + cv * V, s);
  }
}

template <class T>
__global__ void avgpool_bwd_k(const T* __restrict__ dy, T* dx, int acc, int n, int HW, int C) {
  constexpr int V = VecT<T>::N;
  const int CV = C / V;
  const int64_t total = int64_t(n) * HW * CV;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < total; i += int64_t(gridDim.x) * blockDim.x) {
    const int cv = int(i % CV);
    const int64_t pix = i / CV;
    const int nn = int(pix / HW);
    float d[V], o[V];
    ldv(dy + int64_t(nn) * C + cv * V, d);
    if (acc) ldv(dx + pix * C + cv * V, o);
#pragma unroll
    for (int e = 0; e < V; ++e) o[e] = (acc ? o[e] : 0.f) + d[e] / float(HW);
    stv(dx + pix * C + cv * V, o);
  }
}

int ew_grid(int64_t n) {
  int64_t b = (n + kT - 1) / kT;
  return int(b < 148 * 8 ? b : 148 * 8);
}

template <class T>
void partials_launch(int mode, const PieceList& a, const PieceList& b, int C, const float* stats, float* ws,
                     uint64_t ws_bytes, int& G, cudaStream_t st) {
  int64_t total = 0;
  for (int i = 0; i < a.np; ++i) total += a.rows[i];
  const int nseg = mode == 0 ? a.np : (a.np > b.np ? a.np : b.np);
  const int64_t seg_rows = total / nseg;
  const int64_t cap = int64_t((ws_bytes - kTicketBytes) / (2 * uint64_t(C) * sizeof(typename AccOf<T>::type)));
  const int VPR = C / VecT<T>::N;
  const int rpi = kT / VPR;
  int64_t gps = (148 * 4 + nseg - 1) / nseg;
  if (gps * nseg > cap) gps = cap / nseg;
  if (gps > (seg_rows + rpi - 1) / rpi) gps = (seg_rows + rpi - 1) / rpi;
  if (gps < 1) gps = 1;
  G = int(gps * nseg);
  auto* w = reinterpret_cast<typename AccOf<T>::type*>(ws);
  if (mode == 0) bn_partials<T, 0><<<G, kT, 0, st>>>(a, a, C, nseg, int(gps), seg_rows, stats, w);
  else bn_partials<T, 1><<<G, kT, 0, st>>>(a, b, C, nseg, int(gps), seg_rows, stats, w);
}

}  // namespace

// BN kernels need whole 16-byte channel vectors and at most kT vectors per row.
bool bn_supported(int dt, int C) {
  const int V = dt == BF16 ? 8 : 4;
  return C % V == 0 && C / V <= kT;
}

void bn_stats(int dt, const PieceList& x, int C, float eps, float* ws, uint64_t ws_bytes, float* stats,
              cudaStream_t st) {
  int64_t m = 0;
  for (int i = 0; i < x.np; ++i) m += x.rows[i];
  int G = 0;
  if (dt == BF16) {
    partials_launch<bf16>(0, x, x, C, nullptr, ws, ws_bytes, G, st);
    bn_finish_stats<bf16><<<(C + 127) / 128, 128, 0, st>>>(ws, G, C, m, eps, static_cast<const bf16*>(x.ptr[0]), stats);
  } else {
    partials_launch<float>(0, x, x, C, nullptr, ws, ws_bytes, G, st);
    bn_finish_stats<float><<<(C + 127) / 128, 128, 0, st>>>(reinterpret_cast<const double*>(ws), G, C, m, eps, static_cast<const float*>(x.ptr[0]),
                                                              stats);
  }
}

void bn_apply(int dt, const void* x, const float* stats, const void* gamma, const void* beta, void* y, int64_t rows,
              int C, cudaStream_t st) {
  if (dt == BF16) {
    const int64_t nv = rows * C / 8;
    bn_apply_k<bf16><<<ew_grid(nv), kT, 0, st>>>(static_cast<const bf16*>(x), stats, static_cast<const bf16*>(gamma),
                                                 static_cast<const bf16*>(beta), static_cast<bf16*>(y), nv, C);
  } else {
    const int64_t nv = rows * C / 4;
    bn_apply_k<float><<<ew_grid(nv), kT, 0, st>>>(static_cast<const float*>(x), stats,
                                                  static_cast<const float*>(gamma), static_cast<const float*>(beta),
                                                  static_cast<float*>(y), nv, C);
  }
}

void bn_bwd_sums(int dt, const PieceList& dy, const PieceList& x, const void* gamma, int C, float* ws,
                 uint64_t ws_bytes, float* stats, float* dgamma, float* dbeta, int pacc, cudaStream_t st) {
  int G = 0;
  if (dt == BF16) {
    partials_launch<bf16>(1, dy, x, C, stats, ws, ws_bytes, G, st);
    bn_finish_bwd<bf16><<<(C + 127) / 128, 128, 0, st>>>(ws, G, C, static_cast<const bf16*>(gamma), stats, dgamma,
                                                         dbeta, pacc);
  } else {
    partials_launch<float>(1, dy, x, C, stats, ws, ws_bytes, G, st);
    bn_finish_bwd<float><<<(C + 127) / 128, 128, 0, st>>>(reinterpret_cast<const double*>(ws), G, C, static_cast<const float*>(gamma), stats, dgamma,
                                                          dbeta, pacc);
  }
}

void bn_bwd_apply(int dt, const void* dy, const void* x, const float* stats, const void* gamma, void* dx, int acc,
                  int64_t rows, int C, int64_t m_total, cudaStream_t st) {
  const float inv_m = 1.f / float(m_total);
  if (dt == BF16) {
    const int64_t nv = rows * C / 8;
    bn_bwd_apply_k<bf16><<<ew_grid(nv), kT, 0, st>>>(static_cast<const bf16*>(dy), static_cast<const bf16*>(x), stats,
                                                     static_cast<const bf16*>(gamma), static_cast<bf16*>(dx), acc, nv,
                                                     C, inv_m);
  } else {
    const int64_t nv = rows * C / 4;
    bn_bwd_apply_k<float><<<ew_grid(nv), kT, 0, st>>>(static_cast<const float*>(dy), static_cast<const float*>(x),
                                                      stats, static_cast<const float*>(gamma), static_cast<float*>(dx),
                                                      acc, nv, C, inv_m);
  }
}

void maxpool_fwd(int dt, const void* x, void* y, int n, int H, int W, int C, int P, int Q, int k, int stride, int pad,
                 cudaStream_t st) {
  if (dt == BF16)
    maxpool_fwd_k<bf16><<<ew_grid(int64_t(n) * P * Q * C / 8), kT, 0, st>>>(
        static_cast<const bf16*>(x), static_cast<bf16*>(y), n, H, W, C, P, Q, k, stride, pad);
  else
    maxpool_fwd_k<float><<<ew_grid(int64_t(n) * P * Q * C / 4), kT, 0, st>>>(
        static_cast<const float*>(x), static_cast<float*>(y), n, H, W, C, P, Q, k, stride, pad);
}

void maxpool_bwd(int dt, const void* dy, const void* x, void* dx, int acc, int n, int H, int W, int C, int P, int Q,
                 int k, int stride, int pad, cudaStream_t st) {
  if (dt == BF16)
    maxpool_bwd_k<bf16><<<ew_grid(int64_t(n) * H * W * C / 8), kT, 0, st>>>(
        static_cast<const bf16*>(dy), static_cast<const bf16*>(x), static_cast<bf16*>(dx), acc, n, H, W, C, P, Q, k,
        stride, pad);
  else
    maxpool_bwd_k<float><<<ew_grid(int64_t(n) * H * W * C / 4), kT, 0, st>>>(
        static_cast<const float*>(dy), static_cast<const float*>(x), static_cast<float*>(dx), acc, n, H, W, C, P, Q,
        k, stride, pad);
}

void avgpool_fwd(int dt, const void* x, void* y, int n, int HW, int C, cudaStream_t st) {
  if (dt == BF16)
    avgpool_fwd_k<bf16><<<ew_grid(int64_t(n) * C / 8), kT, 0, st>>>(static_cast<const bf16*>(x),
                                                                     static_cast<bf16*>(y), n, HW, C);
  else
    avgpool_fwd_k<float><<<ew_grid(int64_t(n) * C / 4), kT, 0, st>>>(static_cast<const float*>(x),
                                                                      static_cast<float*>(y), n, HW, C);
}

void avgpool_bwd(int dt, const void* dy, void* dx, int acc, int n, int HW, int C, cudaStream_t st) {
  if (dt == BF16)
    avgpool_bwd_k<bf16><<<ew_grid(int64_t(n) * HW * C / 8), kT, 0, st>>>(static_cast<const bf16*>(dy),
                                                                          static_cast<bf16*>(dx), acc, n, HW, C);
  else
    avgpool_bwd_k<float><<<ew_grid(int64_t(n) * HW * C / 4), kT, 0, st>>>(static_cast<const float*>(dy),
                                                                           static_cast<float*>(dx), acc, n, HW, C);
}

}  // namespace tsk
