// Implicit-GEMM convolution on the 5th-generation tensor cores (sm_100a) — the
// conv micro-op of SURVEY.md §8(a) a6/a8 (configs C2 VGG-16, C3 ResNet-50).
//
// The three products of a conv layer are GEMMs over an index map, never a
// materialised im2col buffer (which would be 9x the activation for a 3x3 conv and
// would itself need budget):
//   fprop  Y[m=(n,p,q), k_out]   = sum_{(r,s,c)}  X[n, p*st-pad+r, q*st-pad+s, c] W[k_out,r,s,c]
//   dgrad  dX[m=(n,h,w), c]      = sum_{(r,s,ko)} dY[n, (h+pad-r)/st, (w+pad-s)/st, ko] W[ko,r,s,c]
//                                   (terms whose quotient is fractional or out of range vanish)
//   wgrad  dW^T[m=(r,s,c), ko]   = sum_{(n,p,q)}  X[n, p*st-pad+r, q*st-pad+s, c] dY[n,p,q,ko]
// Four producer warps gather 16-byte channel vectors with cp.async (zero-fill for
// padding, fractional strides and tails) straight into the 128B-swizzled UMMA
// layouts (K-major or MN-major as the source's contiguous dim dictates), release
// each stage to the single-thread tcgen05.mma issuer through an mbarrier after
// a proxy fence, and four epilogue warps drain the double-buffered TMEM
// accumulator.  A micro-op (a block of samples) is the same kernel on a
// shifted pointer with n = its sample count.  wgrad splits its long pixel
// reduction over CTAs (split-K, fp32 red.add), and accumulates across micro-ops
// (merge = sum).
#include <algorithm>

#include "common.cuh"
#include "kernels.h"
#include "tc_ptx.cuh"

namespace tsk {

namespace {

using namespace tc;

constexpr int BM = 128, BK = 64;
constexpr int kEpiWarps = 4, kProdWarps = 4;
constexpr int kMmaWarp = kEpiWarps;      // warp 4
constexpr int kProd0 = kEpiWarps + 1;    // warps 5..8
constexpr int kThreads = 32 * (kEpiWarps + 1 + kProdWarps);
constexpr int kProdThreads = 32 * kProdWarps;
constexpr int kSmemLimit = 232448;

enum Mode : int { FPROP = 1, DGRAD = 2, WGRAD = 3 };

struct CtP {
  int n, H, W, C, K, R, S, P, Q, st, pad;
  const bf16 *x, *w, *dy;
  int M, N, Kg;
  int tiles_m, tiles_n, num_tiles, num_kb, ksplit, kb_per_split, num_units, n_fastest;
  void* out;
  int acc;  // add into out (bf16: load+add+store; f32: red.add when split-K)
  int red;  // f32 out reduced with red.global.add (split-K)
  const bf16* bias;
};

template <int BN>
constexpr int conv_stages() {
  constexpr int stage = (BM + BN) * BK * 2;
  constexpr int n = (kSmemLimit - 2048) / stage;
  return n > 8 ? 8 : n;
}

__device__ __forceinline__ void cp16(uint32_t dst, const void* src, bool ok) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(ok ? 16 : 0) : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void st_shared16(uint32_t dst, uint4 v) {
  asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(dst), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}
// SW128 K-major: row r (128 B of 64 k), 16-byte chunk j
__device__ __forceinline__ uint32_t kmaj(uint32_t base, int r, int j) {
  return base + uint32_t(r) * 128u + (uint32_t(j ^ (r & 7)) << 4);
}
// SW128 MN-major: 64-element MN blocks of 8 KB; k-row kr, 16-byte MN vector v
__device__ __forceinline__ uint32_t mnmaj(uint32_t base, int kr, int v) {
  return base + uint32_t(v >> 3) * 8192u + uint32_t(kr) * 128u + (uint32_t((v & 7) ^ (kr & 7)) << 4);
}
__device__ __forceinline__ uint16_t ldg_u16(const bf16* p) {
  return __ldg(reinterpret_cast<const unsigned short*>(p));
}
__device__ __forceinline__ uint4 pack8(const uint16_t (&e)[8]) {
  return make_uint4(uint32_t(e[0]) | (uint32_t(e[1]) << 16), uint32_t(e[2]) | (uint32_t(e[3]) << 16),
                    uint32_t(e[4]) | (uint32_t(e[5]) << 16), uint32_t(e[6]) | (uint32_t(e[7]) << 16));
}

__device__ __forceinline__ void decode_tile(const CtP& p, int tile, int& m0, int& n0, int BN) {
  int mt, nt;
  if (p.n_fastest) {
    mt = tile / p.tiles_n;
    nt = tile - mt * p.tiles_n;
  } else {
    nt = tile / p.tiles_m;
    mt = tile - nt * p.tiles_m;
  }
  m0 = mt * BM;
  n0 = nt * BN;
}

// ---------------------------------------------------------------- producers
// Each producer thread owns a fixed 16-byte vector column of every tile it fills
// and a strided set of rows, so per-tile index decompositions are hoisted out of
// the K loop and the per-stage work is a handful of adds per cp.async.
template <int MODE, int BN, bool VEC>
struct Producer {
  // ---- per-tile state
  // fprop / dgrad A rows (8 per thread): sample base offset, spatial origin
  int64_t rbase[8];
  int ry[8], rx[8];
  // wgrad A column (r,s,c) per element (8 when scalar)
  int cr[8], cs[8], cc[8];
  bool cok[8];

  __device__ __forceinline__ void tile_setup(const CtP& p, int m0, int tid) {
    if (MODE == FPROP || MODE == DGRAD) {
      const int PQ = MODE == FPROP ? p.P * p.Q : p.H * p.W;
      const int QQ = MODE == FPROP ? p.Q : p.W;
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const int m = m0 + (tid >> 3) + 16 * j;
        if (m < p.M) {
          const int nn = m / PQ, rem = m - nn * PQ, a = rem / QQ, b = rem - a * QQ;
          if (MODE == FPROP) {
            rbase[j] = int64_t(nn) * p.H * p.W * p.C;
            ry[j] = a * p.st - p.pad;
            rx[j] = b * p.st - p.pad;
          } else {
            rbase[j] = int64_t(nn) * p.P * p.Q * p.K;
            ry[j] = a + p.pad;
            rx[j] = b + p.pad;
          }
        } else {
          rbase[j] = 0;
          ry[j] = -(1 << 28);
          rx[j] = -(1 << 28);
        }
      }
    } else {  // WGRAD: A column mn = (r,s,c)
      const int v = tid & 15;
      const int RS = p.R * p.S;
#pragma unroll
      for (int e = 0; e < (VEC ? 1 : 8); ++e) {
        const int mn = m0 + v * 8 + e;
        const int tap = mn / p.C, c = mn - tap * p.C;
        cr[e] = tap / p.S;
        cs[e] = tap - cr[e] * p.S;
        cc[e] = c;
        cok[e] = mn < p.M && tap < RS;
      }
    }
  }

  __device__ __forceinline__ void fill(const CtP& p, uint32_t sa, uint32_t sb, int m0, int n0, int kb, int tid) {
    const int k0 = kb * BK;
    if (MODE == FPROP) {
      const int v = tid & 7;
      // ---- A: im2col of x, K-major
      if (VEC) {
        const int k = k0 + v * 8;
        const bool kok = k < p.Kg;
        const int tap = k / p.C, c = k - tap * p.C;
        const int r = tap / p.S, s = tap - r * p.S;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int ih = ry[j] + r, iw = rx[j] + s;
          const bool ok = kok && unsigned(ih) < unsigned(p.H) && unsigned(iw) < unsigned(p.W);
          const bf16* src = ok ? p.x + rbase[j] + (int64_t(ih) * p.W + iw) * p.C + c : p.x;
          cp16(kmaj(sa, (tid >> 3) + 16 * j, v), src, ok);
        }
      } else {
        int er[8], es[8], ec[8];
        bool eok[8];
#pragma unroll
        for (int e = 0; e < 8; ++e) {
          const int k = k0 + v * 8 + e;
          const int tap = k / p.C;
          ec[e] = k - tap * p.C;
          er[e] = tap / p.S;
          es[e] = tap - er[e] * p.S;
          eok[e] = k < p.Kg;
        }
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          uint16_t el[8];
#pragma unroll
          for (int e = 0; e < 8; ++e) {
            const int ih = ry[j] + er[e], iw = rx[j] + es[e];
            const bool ok = eok[e] && unsigned(ih) < unsigned(p.H) && unsigned(iw) < unsigned(p.W);
            el[e] = ok ? ldg_u16(p.x + rbase[j] + (int64_t(ih) * p.W + iw) * p.C + ec[e]) : uint16_t(0);
          }
          st_shared16(kmaj(sa, (tid >> 3) + 16 * j, v), pack8(el));
        }
      }
      // ---- B: weight rows [K_out, RSC], K-major
#pragma unroll
      for (int j = 0; j < BN / 16; ++j) {
        const int row = (tid >> 3) + 16 * j;
        const int nrow = n0 + row;
        if (VEC) {
          const int k = k0 + v * 8;
          const bool ok = nrow < p.N && k < p.Kg;
          cp16(kmaj(sb, row, v), ok ? p.w + int64_t(nrow) * p.Kg + k : p.w, ok);
        } else {
          uint16_t el[8];
#pragma unroll
          for (int e = 0; e < 8; ++e) {
            const int k = k0 + v * 8 + e;
            el[e] = (nrow < p.N && k < p.Kg) ? ldg_u16(p.w + int64_t(nrow) * p.Kg + k) : uint16_t(0);
          }
          st_shared16(kmaj(sb, row, v), pack8(el));
        }
      }
    } else if (MODE == DGRAD) {
      const int v = tid & 7;
      // ---- A: dY gathered for input pixels, K-major over (r,s,ko)
      {
        const int k = k0 + v * 8;
        const bool kok = k < p.Kg;
        const int tap = k / p.K, ko = k - tap * p.K;
        const int r = tap / p.S, s = tap - r * p.S;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          int ph = ry[j] - r, pw = rx[j] - s;
          bool ok = kok && ph >= 0 && pw >= 0;
          if (p.st != 1) {
            ok = ok && (ph % p.st) == 0 && (pw % p.st) == 0;
            ph /= p.st;
            pw /= p.st;
          }
          ok = ok && ph < p.P && pw < p.Q;
          const bf16* src = ok ? p.dy + rbase[j] + (int64_t(ph) * p.Q + pw) * p.K + ko : p.dy;
          cp16(kmaj(sa, (tid >> 3) + 16 * j, v), src, ok);
        }
      }
      // ---- B: W as [c (MN), (r,s,ko) (K)], MN-major
      {
        constexpr int VPR = BN / 8;          // vectors per k-row
        constexpr int STEP = kProdThreads / VPR;
        const int vv = tid % VPR;
        const int c = n0 + vv * 8;
        const bool cok2 = c < p.N;
        int k = k0 + tid / VPR;
        int tap = k / p.K, ko = k - tap * p.K;
#pragma unroll
        for (int j = 0; j < BK / STEP; ++j) {
          const bool ok = cok2 && k < p.Kg;
          const bf16* src = ok ? p.w + (int64_t(ko) * p.R * p.S + tap) * p.C + c : p.w;
          cp16(mnmaj(sb, tid / VPR + STEP * j, vv), src, ok);
          k += STEP;
          ko += STEP;
          while (ko >= p.K) {
            ko -= p.K;
            ++tap;
          }
        }
      }
    } else {  // WGRAD
      // ---- A: im2col of x over (r,s,c) (MN) x output pixels (K), MN-major
      {
        const int v = tid & 15;
        int pix = k0 + (tid >> 4);
        const int PQ = p.P * p.Q;
        int nn = pix / PQ, rem = pix - nn * PQ;
        int pp = rem / p.Q, qq = rem - pp * p.Q;
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const bool kok = pix < p.Kg;
          const int64_t xb = int64_t(nn) * p.H * p.W * p.C;
          if (VEC) {
            const int ih = pp * p.st - p.pad + cr[0], iw = qq * p.st - p.pad + cs[0];
            const bool ok = kok && cok[0] && unsigned(ih) < unsigned(p.H) && unsigned(iw) < unsigned(p.W);
            const bf16* src = ok ? p.x + xb + (int64_t(ih) * p.W + iw) * p.C + cc[0] : p.x;
            cp16(mnmaj(sa, (tid >> 4) + 8 * j, v), src, ok);
          } else {
            uint16_t el[8];
#pragma unroll
            for (int e = 0; e < 8; ++e) {
              const int ih = pp * p.st - p.pad + cr[e], iw = qq * p.st - p.pad + cs[e];
              const bool ok = kok && cok[e] && unsigned(ih) < unsigned(p.H) && unsigned(iw) < unsigned(p.W);
              el[e] = ok ? ldg_u16(p.x + xb + (int64_t(ih) * p.W + iw) * p.C + cc[e]) : uint16_t(0);
            }
            st_shared16(mnmaj(sa, (tid >> 4) + 8 * j, v), pack8(el));
          }
          pix += 8;
          qq += 8;
          while (qq >= p.Q) {
            qq -= p.Q;
            if (++pp == p.P) {
              pp = 0;
              ++nn;
            }
          }
        }
      }
      // ---- B: dY rows (pixels, K) x k_out (MN), MN-major
      {
        constexpr int VPR = BN / 8;
        constexpr int STEP = kProdThreads / VPR;
        const int vv = tid % VPR;
        const int ko = n0 + vv * 8;
        const bool kok2 = ko < p.N;
#pragma unroll
        for (int j = 0; j < BK / STEP; ++j) {
          const int kr = tid / VPR + STEP * j;
          const int pix = k0 + kr;
          const bool ok = kok2 && pix < p.Kg;
          cp16(mnmaj(sb, kr, vv), ok ? p.dy + int64_t(pix) * p.K + ko : p.dy, ok);
        }
      }
    }
  }
};

template <int MODE, int BN, bool VEC>
__global__ void __launch_bounds__(kThreads, 1) conv_tc_kernel(const CtP p) {
  constexpr int A_BYTES = BM * BK * 2;
  constexpr int B_BYTES = BN * BK * 2;
  constexpr int STAGE = A_BYTES + B_BYTES;
  constexpr int STAGES = conv_stages<BN>();
  // cp.async groups a producer thread keeps in flight before releasing the oldest
  // stage: all but two stages, so each SM has ~150 KB of gathers outstanding (the
  // L2 latency x bandwidth product; fewer leaves the tensor pipe starved)
  constexpr int kLag = STAGES - 2;
  constexpr uint32_t TMEM_COLS = 2 * BN;
  constexpr int A_MN = MODE == WGRAD ? 1 : 0;
  constexpr int B_MN = MODE == FPROP ? 0 : 1;
  constexpr uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | (uint32_t(A_MN) << 15) | (uint32_t(B_MN) << 16) |
                             (uint32_t(BN >> 3) << 17) | (uint32_t(BM >> 4) << 24);

  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + STAGES * STAGE);
  uint64_t* empty = full + STAGES;
  uint64_t* tfull = empty + STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], kProdThreads);
      mbar_init(&empty[s], 1);
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(&tfull[s], 1);
      mbar_init(&tempty[s], 32 * kEpiWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kMmaWarp) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(TMEM_COLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp >= kProd0) {
    // ===== gather producers =====
    const int tid = threadIdx.x - 32 * kProd0;
    Producer<MODE, BN, VEC> pr;
    int stage = 0;
    uint32_t phase = 0;
    int filled = 0;  // stages filled so far; the one kLag fills back is released after each fill
    for (int unit = blockIdx.x; unit < p.num_units; unit += gridDim.x) {
      const int tile = unit / p.ksplit, ks = unit - tile * p.ksplit;
      int m0, n0;
      decode_tile(p, tile, m0, n0, BN);
      pr.tile_setup(p, m0, tid);
      const int kb0 = ks * p.kb_per_split;
      const int kb1 = min(p.num_kb, kb0 + p.kb_per_split);
      for (int kb = kb0; kb < kb1; ++kb) {
        mbar_wait(&empty[stage], phase ^ 1);
        const uint32_t sa = smem_u32(smem + stage * STAGE);
        pr.fill(p, sa, sa + A_BYTES, m0, n0, kb, tid);
        cp_commit();
        if (++filled > kLag) {
          cp_wait<kLag>();
          fence_async_smem();
          mbar_arrive(&full[(stage + STAGES - kLag) % STAGES]);
        }
        if (++stage == STAGES) {
          stage = 0;
          phase ^= 1;
        }
      }
    }
    cp_wait<0>();
    fence_async_smem();
    for (int i = min(filled, kLag); i >= 1; --i) mbar_arrive(&full[(stage + STAGES - i) % STAGES]);
  } else if (warp == kMmaWarp) {
    if (lane == 0) {
      // ===== MMA issuer (single thread) =====
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      constexpr uint32_t a_lbo = A_MN ? 8192 : 16, b_lbo = B_MN ? 8192 : 16;
      constexpr uint32_t a_kstep = A_MN ? 2048 : 32, b_kstep = B_MN ? 2048 : 32;
      for (int unit = blockIdx.x; unit < p.num_units; unit += gridDim.x) {
        const int ks = unit % p.ksplit;
        const int kb0 = ks * p.kb_per_split;
        const int kb1 = min(p.num_kb, kb0 + p.kb_per_split);
        mbar_wait(&tempty[acc], acc_phase ^ 1);
        tc_fence_after();
        const uint32_t tmem_d = tmem_base + uint32_t(acc * BN);
        for (int kb = kb0; kb < kb1; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint32_t sa = smem_u32(smem + stage * STAGE);
          const uint32_t sb = sa + A_BYTES;
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            const uint64_t ad = smem_desc(sa + k * a_kstep, a_lbo, 1024);
            const uint64_t bd = smem_desc(sb + k * b_kstep, b_lbo, 1024);
            tc_mma(tmem_d, ad, bd, idesc, (kb > kb0 || k > 0) ? 1u : 0u);
          }
          tc_commit(&empty[stage]);
          if (++stage == STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
        tc_commit(&tfull[acc]);
        if (++acc == 2) {
          acc = 0;
          acc_phase ^= 1;
        }
      }
    }
  } else {
    // ===== epilogue: TMEM -> registers -> global (warp q owns TMEM lanes 32q..32q+31) =====
    const int q = warp;
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int unit = blockIdx.x; unit < p.num_units; unit += gridDim.x) {
      const int tile = unit / p.ksplit;
      int m0, n0;
      decode_tile(p, tile, m0, n0, BN);
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const int row = m0 + q * 32 + lane;
      const bool row_ok = row < p.M;
#pragma unroll 1
      for (int c = 0; c < BN / 32; ++c) {
        uint32_t r[32];
        tmem_ld32(tmem_base + (uint32_t(q * 32) << 16) + uint32_t(acc * BN + c * 32), r);
        const int col0 = n0 + c * 32;
        if (row_ok && col0 < p.N) {
        const bool full_chunk = col0 + 32 <= p.N;
        if (MODE == WGRAD) {
          // dW[ko, (r,s,c)] with m = (r,s,c): lanes hold consecutive m -> coalesced per column
          float* o = reinterpret_cast<float*>(p.out) + row;
#pragma unroll
          for (int i = 0; i < 32; ++i) {
            if (!full_chunk && col0 + i >= p.N) break;
            float* a = o + int64_t(col0 + i) * p.M;
            const float v = __uint_as_float(r[i]);
            if (p.red) atomicAdd(a, v);
            else if (p.acc) *a += v;
            else *a = v;
          }
        } else {
          bf16* o = reinterpret_cast<bf16*>(p.out) + int64_t(row) * p.N + col0;
          float v[32];
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
          if (MODE == FPROP && p.bias) {
#pragma unroll
            for (int i = 0; i < 32; ++i)
              if (full_chunk || col0 + i < p.N) v[i] += to_f(p.bias[col0 + i]);
          }
          if (full_chunk) {
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              uint4 u;
              if (p.acc) {
                u = *reinterpret_cast<const uint4*>(o + 8 * j);
                const __nv_bfloat162* o2 = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
                for (int h = 0; h < 4; ++h) {
                  float2 f = __bfloat1622float2(o2[h]);
                  v[8 * j + 2 * h] += f.x;
                  v[8 * j + 2 * h + 1] += f.y;
                }
              }
              __nv_bfloat162* w2 = reinterpret_cast<__nv_bfloat162*>(&u);
#pragma unroll
              for (int h = 0; h < 4; ++h) w2[h] = __floats2bfloat162_rn(v[8 * j + 2 * h], v[8 * j + 2 * h + 1]);
              *reinterpret_cast<uint4*>(o + 8 * j) = u;
            }
          } else {
#pragma unroll
            for (int i = 0; i < 32; ++i)
              if (col0 + i < p.N) o[i] = __float2bfloat16_rn(v[i] + (p.acc ? to_f(o[i]) : 0.f));
          }
        }
        }
        __syncwarp();
      }
      tc_fence_before();
      mbar_arrive(&tempty[acc]);
      if (++acc == 2) {
        acc = 0;
        acc_phase ^= 1;
      }
    }
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  if (warp == kMmaWarp) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(TMEM_COLS));
  }
}

int g_sms = 0;

template <int MODE, int BN, bool VEC>
void launch(const CtP& p, cudaStream_t st) {
  constexpr int STAGE = (BM + BN) * BK * 2;
  const int smem = conv_stages<BN>() * STAGE + 1024 + 1024;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(conv_tc_kernel<MODE, BN, VEC>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    attr = true;
  }
  const int grid = p.num_units < g_sms ? p.num_units : g_sms;
  conv_tc_kernel<MODE, BN, VEC><<<grid, kThreads, smem, st>>>(p);
}

template <int MODE, bool VEC>
void launch_bn(int bn, const CtP& p, cudaStream_t st) {
  switch (bn) {
    case 256: launch<MODE, 256, VEC>(p, st); break;
    case 128: launch<MODE, 128, VEC>(p, st); break;
    default: launch<MODE, 64, VEC>(p, st); break;
  }
}

}  // namespace

bool conv_tc(int mode, const ConvArgs& a, void* out, const void* bias, int acc, cudaStream_t st) {
  // 64-channel layers: TMA-fed kernel (conv_tma.cu); the gather kernel covers the rest
  return conv_tma(mode, a, out, bias, acc, st) || conv_gather(mode, a, out, bias, acc, st);
}

bool conv_gather(int mode, const ConvArgs& a, void* out, const void* bias, int acc, cudaStream_t st) {
  if (a.dtype != BF16 || a.n <= 0) return false;
  if (a.K % 8) return false;                             // dY rows / output rows in 16-byte vectors
  const bool vec = a.C % 8 == 0;
  if (mode == DGRAD && !vec) return false;               // dX of a non-vector input (the image) is never needed
  if (g_sms == 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_sms, cudaDevAttrMultiProcessorCount, dev);
    if (g_sms <= 0) return false;
  }
  CtP p;
  p.n = a.n; p.H = a.H; p.W = a.W; p.C = a.C; p.K = a.K; p.R = a.R; p.S = a.S; p.P = a.P; p.Q = a.Q;
  p.st = a.stride; p.pad = a.pad;
  p.x = static_cast<const bf16*>(a.x);
  p.w = static_cast<const bf16*>(a.w);
  p.dy = static_cast<const bf16*>(a.dy);
  p.out = out;
  p.bias = static_cast<const bf16*>(bias);
  p.acc = acc;
  p.red = 0;
  const int64_t RSC = int64_t(a.R) * a.S * a.C;
  int64_t M, N, Kg;
  if (mode == FPROP) { M = int64_t(a.n) * a.P * a.Q; N = a.K; Kg = RSC; }
  else if (mode == DGRAD) { M = int64_t(a.n) * a.H * a.W; N = a.C; Kg = int64_t(a.R) * a.S * a.K; }
  else { M = RSC; N = a.K; Kg = int64_t(a.n) * a.P * a.Q; }
  if (M >= (int64_t(1) << 31) || Kg >= (int64_t(1) << 31)) return false;
  p.M = int(M); p.N = int(N); p.Kg = int(Kg);
  p.num_kb = int((Kg + BK - 1) / BK);
  // tile width by the wave model of gemm_tc (narrow tiles feed the tensor pipe worse)
  int best_bn = 256;
  double best = 1e30;
  for (int bn : {256, 128, 64}) {
    if (bn > 64 && N <= bn / 2) continue;
    const double eff = bn == 256 ? 0.90 : bn == 128 ? 0.65 : 0.45;
    const int64_t tiles = ((M + BM - 1) / BM) * ((N + bn - 1) / bn);
    const double waves = double((tiles + g_sms - 1) / g_sms);
    // wgrad: split-K fills the machine, so the padded work decides; else whole waves
    const double cost = mode == WGRAD ? double(tiles) * bn / eff : waves * (bn / eff);
    if (cost < best - 1e-12) {
      best = cost;
      best_bn = bn;
    }
  }
  p.tiles_m = int((M + BM - 1) / BM);
  p.tiles_n = int((N + best_bn - 1) / best_bn);
  p.num_tiles = p.tiles_m * p.tiles_n;
  p.n_fastest = mode == WGRAD ? 0 : 1;
  p.ksplit = 1;
  if (mode == WGRAD && p.num_tiles < g_sms && p.num_kb >= 8) {
    p.ksplit = std::max(1, std::min(g_sms / p.num_tiles, p.num_kb / 4));
  }
  p.kb_per_split = (p.num_kb + p.ksplit - 1) / p.ksplit;
  p.ksplit = (p.num_kb + p.kb_per_split - 1) / p.kb_per_split;
  p.num_units = p.num_tiles * p.ksplit;
  if (mode == WGRAD && p.ksplit > 1) {
    if (!acc) cudaMemsetAsync(out, 0, size_t(M) * N * 4, st);
    p.red = 1;
  }
  if (mode == FPROP) {
    if (vec) launch_bn<FPROP, true>(best_bn, p, st);
    else launch_bn<FPROP, false>(best_bn, p, st);
  } else if (mode == DGRAD) {
    launch_bn<DGRAD, true>(best_bn, p, st);
  } else {
    if (vec) launch_bn<WGRAD, true>(best_bn, p, st);
    else launch_bn<WGRAD, false>(best_bn, p, st);
  }
  return true;
}

namespace {
void record(int kind, const ConvArgs& a, cudaStream_t st, int tc, GemmRecord& rec, bool begin) {
  auto* sink = gemm_records_sink();
  if (!sink) return;
  if (begin) {
    cudaEventCreate(&rec.start);
    cudaEventCreate(&rec.stop);
    cudaEventRecord(rec.start, st);
    return;
  }
  cudaEventRecord(rec.stop, st);
  rec.flop = 2.0 * double(a.n) * a.P * a.Q * a.K * double(a.R) * a.S * a.C;
  rec.M = kind == WGRAD ? a.R * a.S * a.C : (kind == FPROP ? a.n * a.P * a.Q : a.n * a.H * a.W);
  rec.N = kind == FPROP ? a.K : (kind == DGRAD ? a.C : a.K);
  rec.K = kind == FPROP ? a.R * a.S * a.C : (kind == DGRAD ? a.R * a.S * a.K : a.n * a.P * a.Q);
  rec.batch = 1;
  rec.tc = tc;
  rec.kind = kind;
  sink->push_back(rec);
}
void conv_run(int mode, const ConvArgs& a, void* out, const void* bias, int acc, cudaStream_t st) {
  GemmRecord rec{};
  record(mode, a, st, 0, rec, true);
  int tc = conv_tc(mode, a, out, bias, acc, st) ? 1 : 0;
  if (!tc) conv_simt(mode, a, out, bias, acc, st);
  record(mode, a, st, tc, rec, false);
}
}  // namespace

void conv_fprop(const ConvArgs& a, void* y, const void* bias, cudaStream_t st) { conv_run(FPROP, a, y, bias, 0, st); }
void conv_dgrad(const ConvArgs& a, void* dx, int acc, cudaStream_t st) { conv_run(DGRAD, a, dx, nullptr, acc, st); }
void conv_wgrad(const ConvArgs& a, float* dw, int acc, cudaStream_t st) { conv_run(WGRAD, a, dw, nullptr, acc, st); }

}  // namespace tsk
