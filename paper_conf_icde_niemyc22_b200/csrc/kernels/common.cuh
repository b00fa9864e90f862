// Device helpers shared by the sm_100a kernels.
#pragma once
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdint>

namespace tsk {

typedef __nv_bfloat16 bf16;

__device__ __forceinline__ float to_f(float x) { return x; }
__device__ __forceinline__ float to_f(bf16 x) { return __bfloat162float(x); }
template <class T>
__device__ __forceinline__ T from_f(float x);
template <>
__device__ __forceinline__ float from_f<float>(float x) { return x; }
template <>
__device__ __forceinline__ bf16 from_f<bf16>(float x) { return __float2bfloat16_rn(x); }

// erf-GELU (R16) shared by the elementwise kernels and the GEMM epilogue (one definition, so a
// fused epilogue computes bit-for-bit what the separate kernel would).  erf by Abramowitz &
// Stegun 7.1.26 (|error| <= 1.5e-7) on the MUFU unit: t = rcp.approx(1 + p|z|) and
// exp(-z^2) = ex2.approx(-x^2 log2(e) / 2), which the derivative's normal pdf reuses — about
// 13 FP32 instructions and 2 MUFU per element (the CUDA erff costs ~22 with selects, an IEEE
// reciprocal far more; both made the GELU passes ALU-bound).
__device__ __forceinline__ float ex2_approx(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ float rcp_approx(float x) {
  float y;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
// erf(x / sqrt 2) given e = exp(-x^2 / 2)
__device__ __forceinline__ float erf_gelu(float x, float e) {
  const float t = rcp_approx(fmaf(0.3275911f * 0.70710678118654752f, fabsf(x), 1.f));
  float p = fmaf(1.061405429f, t, -1.453152027f);
  p = fmaf(p, t, 1.421413741f);
  p = fmaf(p, t, -0.284496736f);
  p = fmaf(p, t, 0.254829592f);
  return copysignf(fmaf(-p * t, e, 1.f), x);
}
__device__ __forceinline__ float gelu_f(float x) {
  const float e = ex2_approx(x * x * -0.72134752044448170f);  // exp(-x^2/2) = 2^(-x^2 log2(e)/2)
  return 0.5f * x * (1.f + erf_gelu(x, e));
}
__device__ __forceinline__ float gelu_d(float x) {
  const float e = ex2_approx(x * x * -0.72134752044448170f);
  const float cdf = 0.5f * (1.f + erf_gelu(x, e));
  return fmaf(x * 0.39894228040143268f, e, cdf);
}
__device__ __forceinline__ float bf16_round(float x) { return __bfloat162float(__float2bfloat16_rn(x)); }

// Philox4x32-10 (Salmon et al. SC'11); reading D-RNG: element idx takes the 16-bit half
// (idx & 1) of word ((idx >> 1) & 3) of Philox(counter = (idx>>3 lo, idx>>3 hi, step, 0),
// key = (seed, 0x5453504C)), and is kept when that half >= floor(p * 2^16): one call covers
// eight consecutive elements.
__device__ __forceinline__ uint4 philox4x32_10(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3,
                                               uint32_t k0, uint32_t k1) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    uint32_t hi0 = __umulhi(0xD2511F53u, c0), lo0 = 0xD2511F53u * c0;
    uint32_t hi1 = __umulhi(0xCD9E8D57u, c2), lo1 = 0xCD9E8D57u * c2;
    uint32_t n0 = hi1 ^ c1 ^ k0, n2 = hi0 ^ c3 ^ k1;
    c0 = n0;
    c1 = lo1;
    c2 = n2;
    c3 = lo0;
    k0 += 0x9E3779B9u;
    k1 += 0xBB67AE85u;
  }
  return make_uint4(c0, c1, c2, c3);
}
constexpr uint32_t kPhiloxKey1 = 0x5453504Cu;
// keep bits of the eight elements of one Philox call (bit i = element 8c + i)
__device__ __forceinline__ uint32_t keep_bits8(const uint4& w, uint32_t thr16) {
  return uint32_t((w.x & 0xFFFFu) >= thr16) | (uint32_t((w.x >> 16) >= thr16) << 1) |
         (uint32_t((w.y & 0xFFFFu) >= thr16) << 2) | (uint32_t((w.y >> 16) >= thr16) << 3) |
         (uint32_t((w.z & 0xFFFFu) >= thr16) << 4) | (uint32_t((w.z >> 16) >= thr16) << 5) |
         (uint32_t((w.w & 0xFFFFu) >= thr16) << 6) | (uint32_t((w.w >> 16) >= thr16) << 7);
}
// the 16-bit draw of element idx (one call per element: tails and reference kernels)
__device__ __forceinline__ uint32_t philox_u16(uint64_t idx, uint32_t seed, uint32_t step) {
  const uint64_t c = idx >> 3;
  const uint4 r = philox4x32_10(uint32_t(c), uint32_t(c >> 32), step, 0u, seed, kPhiloxKey1);
  const uint32_t q = uint32_t(idx >> 1) & 3u;
  const uint32_t word = q == 0 ? r.x : q == 1 ? r.y : q == 2 ? r.z : r.w;
  return (idx & 1) ? (word >> 16) : (word & 0xFFFFu);
}
// floor(p * 2^16) (p in [0, 1))
inline uint32_t dropout_thr16(float p) {
  if (p <= 0.f) return 0u;
  const double t = double(p) * 65536.0;
  return t >= 65535.0 ? 65535u : uint32_t(t);
}

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

}  // namespace tsk
