// Vectorised elementwise micro-op kernels (HBM-bound: 16-byte loads/stores,
// grid-stride loops sized to the SM count).  Every kernel takes micro-tensor
// views, so a split micro-op is the same kernel on a shifted pointer; `acc`
// selects accumulate-into-gradient (a later backward op adding its share).
#include "common.cuh"
#include "kernels.h"

namespace tsk {

namespace {

enum EwOp : int { RELU_F, RELU_B, GELU_F, GELU_B, TANH_F, TANH_B, ADD_F, AXPY, DROP };

struct EwP {
  int64_t elem0;
  float p, scale;
  uint32_t seed, step, thr;
  const uint32_t* step_ptr;
};

// GELU: gelu_f / gelu_d from common.cuh (shared with the GEMM epilogue).

template <int OP>
__device__ __forceinline__ float ew_apply(float a, float b, int64_t idx, uint32_t word, const EwP& q) {
  switch (OP) {
    case RELU_F: return fmaxf(a, 0.f);
    case RELU_B: return b > 0.f ? a : 0.f;   // a = dy, b = y
    case GELU_F: return gelu_f(a);
    case GELU_B: return a * gelu_d(b);       // a = dy, b = x
    case TANH_F: return tanhf(a);
    case TANH_B: return a * (1.f - b * b);   // a = dy, b = y
    case ADD_F: return a + b;
    case AXPY: return a;
    case DROP: return word >= q.thr ? a * q.scale : 0.f;
  }
  return 0.f;
}

template <class T, int OP, int V>
__device__ __forceinline__ void ew_vec(const T* __restrict__ a, const T* __restrict__ b, T* y, int64_t v, int acc,
                                       const EwP& q, const T* av, const T* bv, T* yv) {
  uint32_t words[V];  // DROP: the element's 16-bit draw (D-RNG)
  if constexpr (OP == DROP) {
    const int64_t i0 = q.elem0 + v * V;
    if ((i0 & 7) == 0 && V % 8 == 0) {
#pragma unroll
      for (int j = 0; j < V; j += 8) {
        const uint64_t c = uint64_t(i0 + j) >> 3;
        const uint4 r = philox4x32_10(uint32_t(c), uint32_t(c >> 32), q.step, 0u, q.seed, kPhiloxKey1);
        const uint32_t w4[4] = {r.x, r.y, r.z, r.w};
#pragma unroll
        for (int e = 0; e < 8; ++e) words[j + e] = (e & 1) ? (w4[e >> 1] >> 16) : (w4[e >> 1] & 0xFFFFu);
      }
    } else {
#pragma unroll
      for (int j = 0; j < V; ++j) words[j] = philox_u16(uint64_t(i0 + j), q.seed, q.step);
    }
  }
#pragma unroll
  for (int i = 0; i < V; ++i) {
    float r = ew_apply<OP>(to_f(av[i]), b ? to_f(bv[i]) : 0.f, v * V + i, OP == DROP ? words[i] : 0u, q);
    if (acc) r += to_f(yv[i]);
    yv[i] = from_f<T>(r);
  }
}

// U vectors of V elements per thread per iteration, all loads issued before any math,
// so each SM keeps U x 16 B x threads in flight (HBM latency hiding, guide G7).
template <class T, int OP, int V>
__global__ void __launch_bounds__(256) ew_kernel(const T* __restrict__ a, const T* __restrict__ b, T* y, int64_t n,
                                                 int acc, EwP q) {
  constexpr int U = 2;  // two 16-byte vectors in flight per thread (HBM latency)
  if constexpr (OP == DROP)
    if (q.step_ptr) q.step = *q.step_ptr;
  const int64_t nv = n / V;
  const int64_t stride = int64_t(gridDim.x) * blockDim.x;
  for (int64_t v0 = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; v0 < nv; v0 += stride * U) {
    T av[U][V], bv[U][V], yv[U][V];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = v0 + u * stride;
      if (v >= nv) break;
      if constexpr (V * sizeof(T) == 16) {
        *reinterpret_cast<uint4*>(av[u]) = reinterpret_cast<const uint4*>(a)[v];
        if (b) *reinterpret_cast<uint4*>(bv[u]) = reinterpret_cast<const uint4*>(b)[v];
        if (acc) *reinterpret_cast<uint4*>(yv[u]) = reinterpret_cast<const uint4*>(y)[v];
      } else {
#pragma unroll
        for (int i = 0; i < V; ++i) {
          av[u][i] = a[v * V + i];
          if (b) bv[u][i] = b[v * V + i];
          if (acc) yv[u][i] = y[v * V + i];
        }
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t v = v0 + u * stride;
      if (v >= nv) break;
      ew_vec<T, OP, V>(a, b, y, v, acc, q, av[u], bv[u], yv[u]);
      if constexpr (V * sizeof(T) == 16) {
        reinterpret_cast<uint4*>(y)[v] = *reinterpret_cast<uint4*>(yv[u]);
      } else {
#pragma unroll
        for (int i = 0; i < V; ++i) y[v * V + i] = yv[u][i];
      }
    }
  }
  // scalar tail
  for (int64_t i = nv * V + int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += stride) {
    uint32_t w = 0;
    if constexpr (OP == DROP) w = philox_u16(uint64_t(q.elem0 + i), q.seed, q.step);
    float r = ew_apply<OP>(to_f(a[i]), b ? to_f(b[i]) : 0.f, i, w, q);
    if (acc) r += to_f(y[i]);
    y[i] = from_f<T>(r);
  }
}

int g_grid_cap = 0;

template <class T, int OP>
void ew_launch(const void* a, const void* b, void* y, int64_t n, int acc, const EwP& q, cudaStream_t st) {
  if (n <= 0) return;
  if (!g_grid_cap) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    g_grid_cap = sms * 8;
  }
  constexpr int V = 16 / sizeof(T);
  bool aligned = (reinterpret_cast<uintptr_t>(a) % 16 == 0) && (reinterpret_cast<uintptr_t>(y) % 16 == 0) &&
                 (!b || reinterpret_cast<uintptr_t>(b) % 16 == 0);
  int64_t work = aligned ? (n + V - 1) / V : n;
  int grid = int(work / 256 + 1 < g_grid_cap ? work / 256 + 1 : g_grid_cap);
  if (aligned)
    ew_kernel<T, OP, V><<<grid, 256, 0, st>>>((const T*)a, (const T*)b, (T*)y, n, acc, q);
  else
    ew_kernel<T, OP, 1><<<grid, 256, 0, st>>>((const T*)a, (const T*)b, (T*)y, n, acc, q);
}

template <int OP>
void ew(int dt, const void* a, const void* b, void* y, int64_t n, int acc, const EwP& q, cudaStream_t st) {
  if (dt == F32) ew_launch<float, OP>(a, b, y, n, acc, q, st);
  else ew_launch<bf16, OP>(a, b, y, n, acc, q, st);
}

__global__ void sgd_kernel(float* __restrict__ m, const float* __restrict__ g, int64_t n, float lr) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x)
    m[i] -= lr * g[i];
}
__global__ void cast_kernel(const float* __restrict__ s, bf16* __restrict__ d, int64_t n) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x)
    d[i] = __float2bfloat16_rn(s[i]);
}
__global__ void uncast_kernel(const bf16* __restrict__ s, float* __restrict__ d, int64_t n) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x)
    d[i] = __bfloat162float(s[i]);
}
__global__ void step_advance_kernel(uint32_t* c) { *c += 1u; }
__global__ void scale_kernel(float* x, int64_t n, float s) {
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x)
    x[i] *= s;
}
// One launch for the whole optimiser step: block b updates chunk b of one parameter
// (fp32 master -= lr * grad) and, for bf16 graphs, writes the bf16 copy from the
// value still in registers (no second pass over the masters, no per-tensor launches).
__global__ void __launch_bounds__(256) sgd_fused_kernel(const SgdChunk* __restrict__ chunks, char* slab, float lr) {
  const SgdChunk c = chunks[blockIdx.x];
  float* m = reinterpret_cast<float*>(slab + c.m_off);
  const float* g = reinterpret_cast<const float*>(slab + c.g_off);
  bf16* cp = c.c_off != ~0ull ? reinterpret_cast<bf16*>(slab + c.c_off) : nullptr;
  const int64_t nv = c.n / 4;
  for (int64_t v = threadIdx.x; v < nv; v += blockDim.x) {
    float4 mv = reinterpret_cast<float4*>(m)[v];
    const float4 gv = reinterpret_cast<const float4*>(g)[v];
    mv.x -= lr * gv.x;
    mv.y -= lr * gv.y;
    mv.z -= lr * gv.z;
    mv.w -= lr * gv.w;
    reinterpret_cast<float4*>(m)[v] = mv;
    if (cp) {
      __nv_bfloat162 lo = __floats2bfloat162_rn(mv.x, mv.y), hi = __floats2bfloat162_rn(mv.z, mv.w);
      uint2 u;
      u.x = *reinterpret_cast<uint32_t*>(&lo);
      u.y = *reinterpret_cast<uint32_t*>(&hi);
      reinterpret_cast<uint2*>(cp)[v] = u;
    }
  }
  for (int64_t i = nv * 4 + threadIdx.x; i < c.n; i += blockDim.x) {
    m[i] -= lr * g[i];
    if (cp) cp[i] = __float2bfloat16_rn(m[i]);
  }
}

int grid_for(int64_t n) {
  int64_t g = (n + 255) / 256;
  return int(g < 148 * 8 ? (g > 0 ? g : 1) : 148 * 8);
}

}  // namespace

static const EwP kNoP{0, 0.f, 1.f, 0u, 0u, 0u};

void relu_fwd(int dt, const void* x, void* y, int64_t n, cudaStream_t st) { ew<RELU_F>(dt, x, nullptr, y, n, 0, kNoP, st); }
void relu_bwd(int dt, const void* dy, const void* y, void* dx, int acc, int64_t n, cudaStream_t st) {
  ew<RELU_B>(dt, dy, y, dx, n, acc, kNoP, st);
}
void gelu_fwd(int dt, const void* x, void* y, int64_t n, cudaStream_t st) { ew<GELU_F>(dt, x, nullptr, y, n, 0, kNoP, st); }
void gelu_bwd(int dt, const void* dy, const void* x, void* dx, int acc, int64_t n, cudaStream_t st) {
  ew<GELU_B>(dt, dy, x, dx, n, acc, kNoP, st);
}
void tanh_fwd(int dt, const void* x, void* y, int64_t n, cudaStream_t st) { ew<TANH_F>(dt, x, nullptr, y, n, 0, kNoP, st); }
void tanh_bwd(int dt, const void* dy, const void* y, void* dx, int acc, int64_t n, cudaStream_t st) {
  ew<TANH_B>(dt, dy, y, dx, n, acc, kNoP, st);
}
void add_fwd(int dt, const void* a, const void* b, void* y, int64_t n, cudaStream_t st) {
  ew<ADD_F>(dt, a, b, y, n, 0, kNoP, st);
}
void axpy(int dt, const void* dy, void* dx, int acc, int64_t n, cudaStream_t st) {
  ew<AXPY>(dt, dy, nullptr, dx, n, acc, kNoP, st);
}

namespace {
// add backward: dy passes to both inputs' gradients (each overwritten or accumulated), dy read once
template <class T>
__global__ void __launch_bounds__(256) axpy2_kernel(const T* __restrict__ dy, T* d1, int acc1, T* d2, int acc2,
                                                    int64_t n) {
  constexpr int V = 16 / sizeof(T);
  const int64_t nv = n / V, stride = int64_t(gridDim.x) * blockDim.x;
  for (int64_t v = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; v < nv; v += stride) {
    T g[V], o1[V], o2[V];
    *reinterpret_cast<uint4*>(g) = reinterpret_cast<const uint4*>(dy)[v];
    if (acc1) *reinterpret_cast<uint4*>(o1) = reinterpret_cast<const uint4*>(d1)[v];
    if (acc2) *reinterpret_cast<uint4*>(o2) = reinterpret_cast<const uint4*>(d2)[v];
#pragma unroll
    for (int i = 0; i < V; ++i) {
      o1[i] = acc1 ? from_f<T>(to_f(g[i]) + to_f(o1[i])) : g[i];
      o2[i] = acc2 ? from_f<T>(to_f(g[i]) + to_f(o2[i])) : g[i];
    }
    reinterpret_cast<uint4*>(d1)[v] = *reinterpret_cast<uint4*>(o1);
    reinterpret_cast<uint4*>(d2)[v] = *reinterpret_cast<uint4*>(o2);
  }
  for (int64_t i = nv * V + int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < n; i += stride) {
    const float gv = to_f(dy[i]);
    d1[i] = acc1 ? from_f<T>(gv + to_f(d1[i])) : dy[i];
    d2[i] = acc2 ? from_f<T>(gv + to_f(d2[i])) : dy[i];
  }
}
}  // namespace

void axpy2(int dt, const void* dy, void* d1, int acc1, void* d2, int acc2, int64_t n, cudaStream_t st) {
  const bool aligned = ((reinterpret_cast<uintptr_t>(dy) | reinterpret_cast<uintptr_t>(d1) |
                         reinterpret_cast<uintptr_t>(d2)) & 15) == 0;
  if (!aligned || n <= 0) {  // rare: two single-output passes
    axpy(dt, dy, d1, acc1, n, st);
    axpy(dt, dy, d2, acc2, n, st);
    return;
  }
  const int64_t work = n / (dt == F32 ? 4 : 8) + 1;
  const int grid = int(work / 256 + 1 < 148 * 8 ? work / 256 + 1 : 148 * 8);
  if (dt == F32)
    axpy2_kernel<float><<<grid, 256, 0, st>>>((const float*)dy, (float*)d1, acc1, (float*)d2, acc2, n);
  else
    axpy2_kernel<bf16><<<grid, 256, 0, st>>>((const bf16*)dy, (bf16*)d1, acc1, (bf16*)d2, acc2, n);
}
void dropout(int dt, const void* x, void* y, int acc, int64_t n, int64_t elem0, float p, uint32_t seed,
             uint32_t step, const uint32_t* step_ptr, cudaStream_t st) {
  EwP q;
  q.elem0 = elem0;
  q.p = p;
  q.scale = p > 0.f ? 1.f / (1.f - p) : 1.f;
  q.seed = seed;
  q.step = step;
  q.step_ptr = step_ptr;
  q.thr = dropout_thr16(p);
  ew<DROP>(dt, x, nullptr, y, n, acc, q, st);
}
void sgd_update(float* master, const float* grad, int64_t n, float lr, float gscale, cudaStream_t st) {
  sgd_kernel<<<grid_for(n), 256, 0, st>>>(master, grad, n, lr * gscale);
}
void sgd_fused(const SgdChunk* chunks, int n_chunks, char* slab, float lr, float gscale, cudaStream_t st) {
  if (n_chunks > 0) sgd_fused_kernel<<<n_chunks, 256, 0, st>>>(chunks, slab, lr * gscale);
}
void cast_f32_bf16(const float* src, void* dst, int64_t n, cudaStream_t st) {
  cast_kernel<<<grid_for(n), 256, 0, st>>>(src, reinterpret_cast<bf16*>(dst), n);
}
void cast_bf16_f32(const void* src, float* dst, int64_t n, cudaStream_t st) {
  uncast_kernel<<<grid_for(n), 256, 0, st>>>(reinterpret_cast<const bf16*>(src), dst, n);
}
void step_advance(uint32_t* counter, cudaStream_t st) { step_advance_kernel<<<1, 1, 0, st>>>(counter); }
void scale_f32(float* x, int64_t n, float s, cudaStream_t st) { scale_kernel<<<grid_for(n), 256, 0, st>>>(x, n, s); }

}  // namespace tsk
