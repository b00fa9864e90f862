// TMA-fed implicit-GEMM convolution on tcgen05 (sm_100a): the conv micro-op of
// SURVEY.md §8(a) a6/a8 when channels come in 64-wide blocks (every VGG-16 /
// ResNet-50 layer but the image layer; those use the cp.async gather kernel in
// conv_tc.cu).
//
// The GEMM M tile is a spatial box of output pixels — Nt images x Ht rows x Wt
// columns (<= 128 pixels) — so the A operand of one (tap, 64-channel block) step is
// ONE 4-D TMA box of the NHWC activation, shifted by the tap: out-of-bounds
// coordinates zero-fill (= the convolution's padding and tile tails) and the TMA
// element stride equals the conv stride.  One thread feeds the tensor pipe; no
// gather arithmetic remains in the K loop.
//   fprop  A = X box at (c, q0*st-pad+s, p0*st-pad+r, n0), B = W[K, RSC] (2-D map)
//   dgrad  sub-pixel phases (h mod st, w mod st): within a phase only the taps
//          r = (ph+pad) mod st + j*st contribute and dY is a plain shifted box, so a
//          strided dgrad does no multiply-by-zero work; B = W[ko, r, s, c] (3-D map,
//          MN-major).  A phase with no tap writes zeros.
//   wgrad  dW^T[(r,s,c), ko] = sum over 64-pixel boxes of X-box (MN-major) x dY-box
//          (MN-major); split-K over the boxes, fp32 red.add.
// Epilogue: four warps drain the double-buffered TMEM accumulator and scatter rows
// back to their pixels.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <mutex>

#include "common.cuh"
#include "kernels.h"
#include "tc_ptx.cuh"

namespace tsk {

namespace {

using namespace tc;

constexpr int BM = 128, BK = 64;
constexpr int kEpiWarps = 4;
constexpr int kMmaWarp = kEpiWarps;  // warp 4
constexpr int kTmaWarp = kEpiWarps + 1;
constexpr int kThreads = 32 * (kEpiWarps + 2);
constexpr int kSmemLimit = 232448;

enum Mode : int { FPROP = 1, DGRAD = 2, WGRAD = 3 };

struct CvP {
  int n, H, W, C, K, R, S, P, Q, st, pad;
  // spatial box of the M tile (fprop/dgrad) or of the K tile (wgrad, 64 pixels)
  int Nt, Ht, Wt;
  int rows;  // Nt*Ht*Wt
  // phases (dgrad: st*st sub-pixel classes; fprop: 1)
  int nph;
  int ph_h[4], ph_w[4];
  int gP[4], gQ[4];      // grid (in output / phase space) per phase
  int tP[4], tQ[4];      // boxes per grid dim
  int tN;                // boxes along the sample dim
  int tile0[5];          // prefix sum of tiles (M boxes x N tiles) per phase
  int r0[4], s0[4], nr[4], ns[4];  // per phase: first tap and tap counts (step tstep)
  int tstep;
  int cblk;              // 64-blocks per tap along the reduction channel dim
  int M, N;              // wgrad M = RSC; N = output channels of the product
  int tiles_n, tiles_m;
  int num_kb;            // wgrad: pixel boxes
  int ksplit, kb_per_split, num_units;
  void* out;
  int acc, red;
  const bf16* bias;
};

template <int BN>
constexpr int tma_stages() {
  constexpr int stage = (BM + BN) * BK * 2;
  constexpr int n = (kSmemLimit - 2048) / stage;
  return n > 8 ? 8 : n;
}

struct Unit {
  int ph, m0box, n0, kb0, kb1;  // m0box: linear box index within the phase (fprop/dgrad) or m tile (wgrad)
  int bn, bp, bq;               // box coordinates (fprop/dgrad)
};

__device__ __forceinline__ void decode(const CvP& p, int MODE, int unit, Unit& u, int BN) {
  if (MODE == WGRAD) {
    const int tile = unit / p.ksplit, ks = unit - tile * p.ksplit;
    const int nt = tile % p.tiles_n, mt = tile / p.tiles_n;
    u.ph = 0;
    u.m0box = mt;
    u.n0 = nt * BN;
    u.kb0 = ks * p.kb_per_split;
    u.kb1 = min(p.num_kb, u.kb0 + p.kb_per_split);
    return;
  }
  int ph = 0;
  while (ph + 1 < p.nph && unit >= p.tile0[ph + 1]) ++ph;
  const int local = unit - p.tile0[ph];
  const int nt = local % p.tiles_n, mb = local / p.tiles_n;  // N tiles fastest: the A box stays in L2
  u.ph = ph;
  u.m0box = mb;
  u.n0 = nt * BN;
  u.bq = mb % p.tQ[ph];
  u.bp = (mb / p.tQ[ph]) % p.tP[ph];
  u.bn = mb / (p.tQ[ph] * p.tP[ph]);
  u.kb0 = 0;
  u.kb1 = p.nr[ph] * p.ns[ph] * p.cblk;
}

template <int MODE, int BN>
__global__ void __launch_bounds__(kThreads, 1)
    conv_tma_kernel(const __grid_constant__ CUtensorMap mA, const __grid_constant__ CUtensorMap mB, const CvP p) {
  constexpr int A_BYTES = BM * BK * 2;
  constexpr int B_BYTES = BN * BK * 2;
  constexpr int STAGE = A_BYTES + B_BYTES;
  constexpr int STAGES = tma_stages<BN>();
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
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(&tfull[s], 1);
      mbar_init(&tempty[s], 32 * kEpiWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mA)) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&mB)) : "memory");
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

  if (warp == kTmaWarp) {
    if (lane == 0) {
      // ===== TMA producer (single thread) =====
      int stage = 0;
      uint32_t phase = 0;
      for (int unit = blockIdx.x; unit < p.num_units; unit += gridDim.x) {
        Unit u;
        decode(p, MODE, unit, u, BN);
        for (int kb = u.kb0; kb < u.kb1; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          uint8_t* sa = smem + stage * STAGE;
          uint8_t* sb = sa + A_BYTES;
          if (MODE == FPROP || MODE == DGRAD) {
            const int tap = kb / p.cblk, cb = kb - tap * p.cblk;
            const int tr = tap / p.ns[u.ph], ts = tap - tr * p.ns[u.ph];
            const int r = p.r0[u.ph] + tr * p.tstep, s = p.s0[u.ph] + ts * p.tstep;
            const int n0 = u.bn * p.Nt, p0 = u.bp * p.Ht, q0 = u.bq * p.Wt;
            const uint32_t bytes = uint32_t(p.rows) * 128u + uint32_t(B_BYTES);
            mbar_arrive_tx(&full[stage], bytes);
            if (MODE == FPROP) {
              tma_load(sa, &mA, &full[stage], cb * 64, q0 * p.st - p.pad + s, p0 * p.st - p.pad + r, n0);
              tma_load(sb, &mB, &full[stage], (r * p.S + s) * p.C + cb * 64, u.n0, 0, 0);
            } else {
              const int dh = (p.ph_h[u.ph] + p.pad - r) / p.st, dw = (p.ph_w[u.ph] + p.pad - s) / p.st;
              tma_load(sa, &mA, &full[stage], cb * 64, q0 + dw, p0 + dh, n0);
#pragma unroll
              for (int i = 0; i < BN / 64; ++i)
                tma_load(sb + i * 8192, &mB, &full[stage], u.n0 + 64 * i, r * p.S + s, cb * 64, 0);
            }
          } else {  // WGRAD: K step = one 64-pixel box
            const int bq = kb % p.tQ[0], bp = (kb / p.tQ[0]) % p.tP[0], bn = kb / (p.tQ[0] * p.tP[0]);
            const int n0 = bn * p.Nt, p0 = bp * p.Ht, q0 = bq * p.Wt;
            int nA = 0;
            int rr[2], ss[2], cc[2];
#pragma unroll
            for (int j = 0; j < 2; ++j) {
              const int mn = u.m0box * BM + 64 * j;
              if (mn < p.M) {
                const int tap = mn / p.C;
                cc[nA] = mn - tap * p.C;
                rr[nA] = tap / p.S;
                ss[nA] = tap - rr[nA] * p.S;
                ++nA;
              }
            }
            int nB = 0;
#pragma unroll
            for (int i = 0; i < BN / 64; ++i)
              if (u.n0 + 64 * i < p.N) ++nB;
            mbar_arrive_tx(&full[stage], uint32_t(nA + nB) * uint32_t(p.rows) * 128u);
            for (int j = 0; j < nA; ++j)
              tma_load(sa + j * 8192, &mA, &full[stage], cc[j], q0 * p.st - p.pad + ss[j],
                       p0 * p.st - p.pad + rr[j], n0);
            for (int i = 0; i < nB; ++i) tma_load(sb + i * 8192, &mB, &full[stage], u.n0 + 64 * i, q0, p0, n0);
          }
          if (++stage == STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
      }
    }
  } else if (warp == kMmaWarp) {
    if (lane == 0) {
      // ===== MMA issuer (single thread) =====
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      constexpr uint32_t a_lbo = A_MN ? 8192 : 16, b_lbo = B_MN ? 8192 : 16;
      // MN-major K step of 16 = 16 k-rows = +2048 B (wgrad k-rows are pixels, 128 B each)
      constexpr uint32_t a_kstep = A_MN ? 2048 : 32, b_kstep = B_MN ? 2048 : 32;
      for (int unit = blockIdx.x; unit < p.num_units; unit += gridDim.x) {
        Unit u;
        decode(p, MODE, unit, u, BN);
        mbar_wait(&tempty[acc], acc_phase ^ 1);
        tc_fence_after();
        const uint32_t tmem_d = tmem_base + uint32_t(acc * BN);
        for (int kb = u.kb0; kb < u.kb1; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint32_t sa = smem_u32(smem + stage * STAGE);
          const uint32_t sb = sa + A_BYTES;
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            const uint64_t ad = smem_desc(sa + k * a_kstep, a_lbo, 1024);
            const uint64_t bd = smem_desc(sb + k * b_kstep, b_lbo, 1024);
            tc_mma(tmem_d, ad, bd, idesc, (kb > u.kb0 || k > 0) ? 1u : 0u);
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
    // ===== epilogue =====
    const int q = warp;
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int unit = blockIdx.x; unit < p.num_units; unit += gridDim.x) {
      Unit u;
      decode(p, MODE, unit, u, BN);
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const int i = q * 32 + lane;  // accumulator row
      const bool no_k = u.kb1 <= u.kb0;
      int64_t obase = -1;           // element offset of this row's output pixel (fprop/dgrad)
      if (MODE != WGRAD) {
        const int hw = p.Ht * p.Wt;
        const int nn = i / hw, rem = i - nn * hw, hh = rem / p.Wt, ww = rem - hh * p.Wt;
        const int n = u.bn * p.Nt + nn, a = u.bp * p.Ht + hh, b = u.bq * p.Wt + ww;
        if (i < p.rows && n < p.n && a < p.gP[u.ph] && b < p.gQ[u.ph]) {
          if (MODE == FPROP) {
            obase = ((int64_t(n) * p.P + a) * p.Q + b) * p.K;
          } else {
            const int h = a * p.st + p.ph_h[u.ph], w = b * p.st + p.ph_w[u.ph];
            obase = ((int64_t(n) * p.H + h) * p.W + w) * p.C;
          }
        }
      }
      const int mrow = u.m0box * BM + i;  // wgrad row = (r,s,c)
#pragma unroll 1
      for (int c = 0; c < BN / 32; ++c) {
        uint32_t r[32];
        tmem_ld32(tmem_base + (uint32_t(q * 32) << 16) + uint32_t(acc * BN + c * 32), r);
        const int col0 = u.n0 + c * 32;
        if (MODE == WGRAD) {
          if (mrow < p.M && col0 < p.N && !no_k) {
            float* o = reinterpret_cast<float*>(p.out) + mrow;
#pragma unroll
            for (int j = 0; j < 32; ++j) {
              if (col0 + j < p.N) {
                float* a = o + int64_t(col0 + j) * p.M;
                const float v = __uint_as_float(r[j]);
                if (p.red) atomicAdd(a, v);
                else if (p.acc) *a += v;
                else *a = v;
              }
            }
          }
        } else if (obase >= 0 && col0 < p.N && !(no_k && p.acc)) {
          // N is a multiple of 64 here, so every 32-column chunk is whole and 16-byte aligned
          bf16* o = reinterpret_cast<bf16*>(p.out) + obase + col0;
          float v[32];
#pragma unroll
          for (int j = 0; j < 32; ++j) v[j] = no_k ? 0.f : __uint_as_float(r[j]);
          if (MODE == FPROP && p.bias) {
#pragma unroll
            for (int j = 0; j < 32; ++j) v[j] += to_f(p.bias[col0 + j]);
          }
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            uint4 w4;
            if (p.acc) {
              w4 = *reinterpret_cast<const uint4*>(o + 8 * j);
              const __nv_bfloat162* o2 = reinterpret_cast<const __nv_bfloat162*>(&w4);
#pragma unroll
              for (int h = 0; h < 4; ++h) {
                float2 f = __bfloat1622float2(o2[h]);
                v[8 * j + 2 * h] += f.x;
                v[8 * j + 2 * h + 1] += f.y;
              }
            }
            __nv_bfloat162* w2 = reinterpret_cast<__nv_bfloat162*>(&w4);
#pragma unroll
            for (int h = 0; h < 4; ++h) w2[h] = __floats2bfloat162_rn(v[8 * j + 2 * h], v[8 * j + 2 * h + 1]);
            *reinterpret_cast<uint4*>(o + 8 * j) = w4;
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

// ------------------------------------------------------------------------- host
PFN_cuTensorMapEncodeTiled_v12000 encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    cudaDriverEntryPointQueryResult q;
    void* f = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(f);
  });
  return fn;
}

// 4-D bf16 map, dims d[0..3] (d[0] contiguous), byte strides s[0..2] of dims 1..3,
// box b[0..3], element strides e[0..3], 128-byte swizzle (inner box = 64 elements).
bool map4(CUtensorMap* m, const void* ptr, const uint64_t d[4], const uint64_t s[3], const uint32_t b[4],
          const uint32_t e[4]) {
  auto fn = encode();
  if (!fn || reinterpret_cast<uintptr_t>(ptr) % 16) return false;
  for (int i = 0; i < 3; ++i)
    if (s[i] % 16) return false;
  for (int i = 0; i < 4; ++i)
    if (b[i] < 1 || b[i] > 256 || d[i] < 1) return false;
  cuuint64_t dims[4] = {d[0], d[1], d[2], d[3]};
  cuuint64_t str[3] = {s[0], s[1], s[2]};
  cuuint32_t box[4] = {b[0], b[1], b[2], b[3]};
  cuuint32_t es[4] = {e[0], e[1], e[2], e[3]};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(ptr), dims, str, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Pixel box of at most `cap` pixels over an (n, P, Q) grid, maximising the useful
// fraction of cap-row tiles; ties go to wider boxes (longer contiguous runs).
void pick_box(int n, int P, int Q, int cap, int st, int& Nt, int& Ht, int& Wt) {
  double best = -1;
  Nt = Ht = Wt = 1;
  for (int wt = 1; wt <= std::min(Q, cap); ++wt) {
    if (wt * st > 256) break;
    for (int ht = 1; ht <= std::min(P, cap / wt); ++ht) {
      if (ht * st > 256) break;
      int nt = std::min(n, cap / (wt * ht));
      if (nt > 256) nt = 256;
      const double tiles = double((n + nt - 1) / nt) * ((P + ht - 1) / ht) * ((Q + wt - 1) / wt);
      const double util = double(n) * P * Q / (tiles * cap);
      if (util > best + 1e-9 || (std::fabs(util - best) <= 1e-9 && wt > Wt)) {
        best = util;
        Nt = nt;
        Ht = ht;
        Wt = wt;
      }
    }
  }
}

// wgrad K tiles: exactly 64 pixels, power-of-two sides — box rows beyond the grid
// read dY out of bounds (zero), so the reduction never sees a stale shared-memory row.
void pick_box64(int n, int P, int Q, int st, int& Nt, int& Ht, int& Wt) {
  double best = -1;
  for (int wt = 1; wt <= 64; wt *= 2)
    for (int ht = 1; wt * ht <= 64; ht *= 2) {
      const int nt = 64 / (wt * ht);
      if (wt * st > 256 || ht * st > 256) continue;
      const double tiles = double((n + nt - 1) / nt) * ((P + ht - 1) / ht) * ((Q + wt - 1) / wt);
      const double util = double(n) * P * Q / (tiles * 64);
      if (util > best + 1e-9 || (std::fabs(util - best) <= 1e-9 && wt > Wt)) {
        best = util;
        Nt = nt;
        Ht = ht;
        Wt = wt;
      }
    }
}

int g_sms = 0;

template <int MODE, int BN>
void launch(const CUtensorMap& a, const CUtensorMap& b, const CvP& p, cudaStream_t st) {
  constexpr int STAGE = (BM + BN) * BK * 2;
  const int smem = tma_stages<BN>() * STAGE + 2048;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(conv_tma_kernel<MODE, BN>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    attr = true;
  }
  const int grid = p.num_units < g_sms ? p.num_units : g_sms;
  conv_tma_kernel<MODE, BN><<<grid, kThreads, smem, st>>>(a, b, p);
}

template <int MODE>
void launch_bn(int bn, const CUtensorMap& a, const CUtensorMap& b, const CvP& p, cudaStream_t st) {
  switch (bn) {
    case 256: launch<MODE, 256>(a, b, p, st); break;
    case 128: launch<MODE, 128>(a, b, p, st); break;
    default: launch<MODE, 64>(a, b, p, st); break;
  }
}

}  // namespace

bool conv_tma(int mode, const ConvArgs& a, void* out, const void* bias, int acc, cudaStream_t st) {
  if (a.dtype != BF16 || a.n <= 0 || a.C % 64 || a.K % 64 || a.stride < 1 || a.stride > 2) return false;
  if (a.pad >= a.R || a.pad >= a.S) return false;
  if (g_sms == 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_sms, cudaDevAttrMultiProcessorCount, dev);
    if (g_sms <= 0) return false;
  }
  CvP p{};
  p.n = a.n; p.H = a.H; p.W = a.W; p.C = a.C; p.K = a.K; p.R = a.R; p.S = a.S; p.P = a.P; p.Q = a.Q;
  p.st = a.stride; p.pad = a.pad;
  p.out = out;
  p.acc = acc;
  p.bias = static_cast<const bf16*>(bias);
  const uint64_t es = 2;
  const uint64_t xd[4] = {uint64_t(a.C), uint64_t(a.W), uint64_t(a.H), uint64_t(a.n)};
  const uint64_t xs[3] = {a.C * es, uint64_t(a.W) * a.C * es, uint64_t(a.H) * a.W * a.C * es};
  const uint64_t yd[4] = {uint64_t(a.K), uint64_t(a.Q), uint64_t(a.P), uint64_t(a.n)};
  const uint64_t ys[3] = {a.K * es, uint64_t(a.Q) * a.K * es, uint64_t(a.P) * a.Q * a.K * es};
  const int RS = a.R * a.S;
  const int64_t RSC = int64_t(RS) * a.C;
  CUtensorMap mA, mB;
  int bn;
  auto pick_bn = [&](int64_t Mrows, int64_t N) {
    int best_bn = 256;
    double best = 1e30;
    for (int b : {256, 128, 64}) {
      if (b > 64 && N <= b / 2) continue;
      const double eff = b == 256 ? 0.90 : b == 128 ? 0.65 : 0.45;
      const int64_t tiles = ((Mrows + BM - 1) / BM) * ((N + b - 1) / b);
      const double waves = double((tiles + g_sms - 1) / g_sms);
      const double cost = waves * (b / eff);
      if (cost < best - 1e-12) {
        best = cost;
        best_bn = b;
      }
    }
    return best_bn;
  };
  if (mode == FPROP || mode == DGRAD) {
    p.tstep = mode == FPROP ? 1 : a.stride;
    p.nph = mode == FPROP ? 1 : a.stride * a.stride;
    for (int ph = 0; ph < p.nph; ++ph) {
      const int hph = ph / a.stride, wph = ph % a.stride;
      p.ph_h[ph] = mode == FPROP ? 0 : hph;
      p.ph_w[ph] = mode == FPROP ? 0 : wph;
      if (mode == FPROP) {
        p.gP[ph] = a.P;
        p.gQ[ph] = a.Q;
        p.r0[ph] = p.s0[ph] = 0;
        p.nr[ph] = a.R;
        p.ns[ph] = a.S;
      } else {
        p.gP[ph] = (a.H - hph + a.stride - 1) / a.stride;
        p.gQ[ph] = (a.W - wph + a.stride - 1) / a.stride;
        p.r0[ph] = (hph + a.pad) % a.stride;
        p.s0[ph] = (wph + a.pad) % a.stride;
        p.nr[ph] = p.r0[ph] < a.R ? (a.R - p.r0[ph] + a.stride - 1) / a.stride : 0;
        p.ns[ph] = p.s0[ph] < a.S ? (a.S - p.s0[ph] + a.stride - 1) / a.stride : 0;
      }
    }
    pick_box(a.n, p.gP[0], p.gQ[0], BM, mode == FPROP ? a.stride : 1, p.Nt, p.Ht, p.Wt);
    p.rows = p.Nt * p.Ht * p.Wt;
    p.N = mode == FPROP ? a.K : a.C;
    p.cblk = (mode == FPROP ? a.C : a.K) / 64;
    const int64_t mrows_est = int64_t(a.n) * (mode == FPROP ? int64_t(a.P) * a.Q : int64_t(a.H) * a.W);
    bn = pick_bn(mrows_est * BM / p.rows, p.N);
    p.tiles_n = (p.N + bn - 1) / bn;
    p.tN = (a.n + p.Nt - 1) / p.Nt;
    p.tile0[0] = 0;
    for (int ph = 0; ph < p.nph; ++ph) {
      p.tP[ph] = (p.gP[ph] + p.Ht - 1) / p.Ht;
      p.tQ[ph] = (p.gQ[ph] + p.Wt - 1) / p.Wt;
      p.tile0[ph + 1] = p.tile0[ph] + p.tN * p.tP[ph] * p.tQ[ph] * p.tiles_n;
    }
    p.num_units = p.tile0[p.nph];
    p.ksplit = 1;
    if (mode == FPROP) {
      const uint32_t box[4] = {64, uint32_t(p.Wt * a.stride), uint32_t(p.Ht * a.stride), uint32_t(p.Nt)};
      const uint32_t e[4] = {1, uint32_t(a.stride), uint32_t(a.stride), 1};
      const uint64_t wd[4] = {uint64_t(RSC), uint64_t(a.K), 1, 1};
      const uint64_t wsr[3] = {RSC * es, RSC * a.K * es, RSC * a.K * es};
      const uint32_t wb[4] = {64, uint32_t(bn), 1, 1}, one[4] = {1, 1, 1, 1};
      if (!map4(&mA, a.x, xd, xs, box, e) || !map4(&mB, a.w, wd, wsr, wb, one)) return false;
    } else {
      const uint32_t box[4] = {64, uint32_t(p.Wt), uint32_t(p.Ht), uint32_t(p.Nt)}, one[4] = {1, 1, 1, 1};
      // W[ko, r, s, c] as (c, tap, ko): box 64 c x 1 tap x 64 ko
      const uint64_t wd[4] = {uint64_t(a.C), uint64_t(RS), uint64_t(a.K), 1};
      const uint64_t wsr[3] = {a.C * es, RSC * es, RSC * a.K * es};
      const uint32_t wb[4] = {64, 1, 64, 1};
      if (!map4(&mA, a.dy, yd, ys, box, one) || !map4(&mB, a.w, wd, wsr, wb, one)) return false;
    }
  } else {  // WGRAD
    p.nph = 1;
    p.M = int(RSC);
    p.N = a.K;
    pick_box64(a.n, a.P, a.Q, a.stride, p.Nt, p.Ht, p.Wt);
    p.rows = p.Nt * p.Ht * p.Wt;
    p.gP[0] = a.P;
    p.gQ[0] = a.Q;
    p.tP[0] = (a.P + p.Ht - 1) / p.Ht;
    p.tQ[0] = (a.Q + p.Wt - 1) / p.Wt;
    p.tN = (a.n + p.Nt - 1) / p.Nt;
    p.num_kb = p.tN * p.tP[0] * p.tQ[0];
    // padded work decides (split-K fills the machine)
    bn = 256;
    double best = 1e30;
    for (int b : {256, 128, 64}) {
      if (b > 64 && p.N <= b / 2) continue;
      const double eff = b == 256 ? 0.90 : b == 128 ? 0.65 : 0.45;
      const double cost = double((p.M + BM - 1) / BM) * ((p.N + b - 1) / b) * b / eff;
      if (cost < best - 1e-12) {
        best = cost;
        bn = b;
      }
    }
    p.tiles_m = (p.M + BM - 1) / BM;
    p.tiles_n = (p.N + bn - 1) / bn;
    const int tiles = p.tiles_m * p.tiles_n;
    p.ksplit = 1;
    if (tiles < g_sms && p.num_kb >= 8) p.ksplit = std::max(1, std::min(g_sms / tiles, p.num_kb / 4));
    p.kb_per_split = (p.num_kb + p.ksplit - 1) / p.ksplit;
    p.ksplit = (p.num_kb + p.kb_per_split - 1) / p.kb_per_split;
    p.num_units = tiles * p.ksplit;
    const uint32_t xb[4] = {64, uint32_t(p.Wt * a.stride), uint32_t(p.Ht * a.stride), uint32_t(p.Nt)};
    const uint32_t e[4] = {1, uint32_t(a.stride), uint32_t(a.stride), 1};
    const uint32_t yb[4] = {64, uint32_t(p.Wt), uint32_t(p.Ht), uint32_t(p.Nt)}, one[4] = {1, 1, 1, 1};
    if (!map4(&mA, a.x, xd, xs, xb, e) || !map4(&mB, a.dy, yd, ys, yb, one)) return false;
    if (p.ksplit > 1) {
      if (!acc) cudaMemsetAsync(out, 0, size_t(p.M) * p.N * 4, st);
      p.red = 1;
    }
  }
  if (p.num_units <= 0) return false;
  if (mode == FPROP) launch_bn<FPROP>(bn, mA, mB, p, st);
  else if (mode == DGRAD) launch_bn<DGRAD>(bn, mA, mB, p, st);
  else launch_bn<WGRAD>(bn, mA, mB, p, st);
  return true;
}

}  // namespace tsk
