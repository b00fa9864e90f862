// bf16 GEMM on the 5th-generation tensor cores (sm_100a): TMA loads into
// 128B-swizzled shared memory, tcgen05.mma issued by one thread with the fp32
// accumulator in TMEM (double-buffered so the epilogue of tile t overlaps the
// MMAs of tile t+1), warp-specialised persistent CTAs (one per SM).
//
// Used for every dense contraction of a micro-op: Linear
// fwd (Y = X W^T), dX = dY W, dW = dY^T X (fp32 out, beta = 1 accumulates across
// splits in ascending k, P:L260 merge-by-sum), and the per-(sample, head)
// attention products.  Operands are strided micro-tensor views: a 4-D TMA map
// (contiguous dim, row dim, batch1, batch2) describes each one, so no copy ever
// materialises a split or a per-head transpose.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <atomic>
#include <cstring>
#include <cstdio>
#include <mutex>

#include "common.cuh"
#include "kernels.h"
#include "tc_ptx.cuh"

namespace tsk {

namespace {

using namespace tc;

constexpr int BM = 128, BK = 64;
// epilogue warps EW: 8 (two per TMEM lane quarter) for plain epilogues; 16 for the fused GELU
// forward epilogue, whose ALU work needs four warps per scheduler to hide its latency
template <int EW>
constexpr int num_threads() { return 64 + 32 * EW; }  // warp0 TMA, warp1 MMA, warps 2.. epilogue

struct TcParams {
  int M, N, K, nb1, nb2;
  int bm;  // output rows per work unit: BM (one CTA) or 2 BM (a CTA pair, cta_group::2)
  int tiles_m, tiles_n, num_tiles, num_kb;
  int n_fastest;  // 1: consecutive tiles walk N (A, the larger operand, is streamed once)
  int ksplit, kb_per_split, num_units;  // work unit = (tile, K slice)
  int split_from;  // units >= split_from are half-width tail units (2 per tile, ksplit == 1)
  int a_mn, b_mn;
  void* C;
  int64_t ldc, cbs1, cbs2;
  int c_f32;
  float alpha, beta;
  const void* bias;
  int bias_f32;
  int tma_store;   // 1: stage in smem and TMA-store; 0: direct per-thread stores
  int reduce_add;  // 1: TMA reduce-add into an fp32 C (beta = 1 or split-K)
  int epi;         // GemmArgs::epi (bf16 TMA-store path only): 1 GELU fwd (2nd output via tmC2), 2 GELU bwd
  const bf16* aux; // epi 2: U, row-major with leading dimension ldaux
  int64_t ldaux;
  // grouped product (GemmArgs::groups): gdim 1 = N groups (B, C, bias per group), 2 = K
  // groups (A, B per group, summed), 3 = M groups (A, C per group); gsize = extent of
  // one group along gdim (a multiple of the tile along it)
  int gdim, gsize;
  const void* bias_g[kMaxGroups];
};
// operand / output tensor maps (one per group; a plain product uses index 0)
struct TmSet {
  CUtensorMap a[kMaxGroups], b[kMaxGroups], c[kMaxGroups], c2;
};
// epilogue staging: per warp, 32x32 output blocks (two for bf16; one for fp32, whose
// products have long K and keep the smem for a deeper operand pipeline)
// (the 16-warp fused epilogues double-buffer too when the CTA stages at most 128 B rows — a CTA
// pair's half tile — so the smem still holds five operand stages: U's store then never waits
// for the previous store's smem read before gelu(U) is staged)
template <bool F32OUT, int EW, int BNL>
constexpr int staging_nbuf() { return (!F32OUT && (EW == 8 || BNL <= 128)) ? 2 : 1; }
constexpr int kSmemLimit = 232448;  // 227 KB opt-in dynamic shared memory per CTA
template <bool F32OUT, int EW, int BNL>
constexpr int staging_bytes() { return EW * staging_nbuf<F32OUT, EW, BNL>() * 32 * 32 * (F32OUT ? 4 : 2); }
template <int BN, bool F32OUT, int EW>
constexpr int num_stages() {
  constexpr int stage = (BM + BN) * BK * 2;
  constexpr int n = (kSmemLimit - staging_bytes<F32OUT, EW, BN>() - 2048) / stage;
  return n > 8 ? 8 : n;
}

// Work unit -> (tile, K slice, half).  The last partial wave's tiles (tiles >= split_from)
// run as two half-width units each (half = 0 / 1 selects the columns), so the tail wave
// of e.g. 512 tiles on 148 SMs costs half a wave instead of a whole one.
__device__ __forceinline__ void decode_unit(const TcParams& p, int unit, int& tile, int& ks, int& hsel) {
  if (unit < p.split_from) {
    tile = unit / p.ksplit;
    ks = unit - tile * p.ksplit;
    hsel = -1;
  } else {
    const int j = unit - p.split_from;
    tile = p.split_from + (j >> 1);
    ks = 0;
    hsel = j & 1;
  }
}

__device__ __forceinline__ void decode_tile(const TcParams& p, int tile, int& b1, int& b2, int& m0, int& n0) {
  int per = p.tiles_m * p.tiles_n;
  int bb = tile / per;
  int r = tile - bb * per;
  // walk the smaller operand's tiles fastest so the larger one streams from DRAM once
  // while the smaller stays in L2
  int nt, mt;
  if (p.n_fastest) {
    mt = r / p.tiles_n;
    nt = r - mt * p.tiles_n;
  } else {
    nt = r / p.tiles_m;
    mt = r - nt * p.tiles_m;
  }
  b1 = bb % p.nb1;
  b2 = bb / p.nb1;
  m0 = mt * p.bm;
  n0 = nt;  // scaled by BN by the caller
}

// CG = 1: one CTA per 128 x BN output tile.  CG = 2: a CTA pair (2-CTA cluster on one
// TPC) computes a 256 x BN tile with tcgen05.mma.cta_group::2 issued by the leader
// (rank 0): each CTA stages its own 128 rows of A and half (BN/2 rows) of B, so the
// pair reads B once for 256 rows and each SM's smem feeds half the B bytes per MMA;
// both CTAs' TMA bytes complete on the leader's full barrier, MMA commits multicast
// to both CTAs' empty/tfull barriers, and each CTA's epilogue drains its own TMEM
// (128 lanes x BN columns) and arrives on the leader's tempty barrier.
template <int BN, bool F32OUT, int EW, int CG>
__global__ void __launch_bounds__(num_threads<EW>(), 1)
    gemm_tc_kernel(const __grid_constant__ TmSet tm, const TcParams p) {
  constexpr int BNL = BN / CG;  // B rows staged by this CTA
  constexpr int A_BYTES = BM * BK * 2;
  constexpr int B_BYTES = BNL * BK * 2;
  constexpr int STAGE = A_BYTES + B_BYTES;
  constexpr int STAGES = num_stages<BNL, F32OUT, EW>();
  constexpr uint32_t TMEM_COLS = 2 * BN;
  constexpr int BUF = 32 * 32 * (F32OUT ? 4 : 2);
  // instruction descriptor: D f32, A/B bf16, M = 128 CG, N = BN
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | (uint32_t(p.a_mn) << 15) |
                         (uint32_t(p.b_mn) << 16) | (uint32_t(BN >> 3) << 17) | (uint32_t((BM * CG) >> 4) << 24);
  // half-width tail units: N = BN / 2
  const uint32_t idesc_h = (idesc & ~(0x3Fu << 17)) | (uint32_t(BN >> 4) << 17);
  const uint32_t rank = CG == 2 ? cluster_ctarank() : 0u;  // rows rank*128.. of the unit
  const int cid = blockIdx.x / CG, ncl = gridDim.x / CG;     // cluster = consecutive blocks

  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + STAGES * STAGE);
  uint64_t* empty = full + STAGES;
  uint64_t* tfull = empty + STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);
  uint8_t* cstage = smem + STAGES * STAGE + 1024;  // 1024-aligned epilogue staging

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 0 && lane == 0) {
    for (int s = 0; s < STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int s = 0; s < 2; ++s) {
      mbar_init(&tfull[s], 1);
      mbar_init(&tempty[s], EW * CG);  // one arrive per epilogue warp of each CTA
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tm.a[0])) : "memory");
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tm.b[0])) : "memory");
  }
  if (warp == 1) {
    if constexpr (CG == 1) {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                   "r"(TMEM_COLS));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    } else {
      asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                   "r"(TMEM_COLS));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    }
  }
  tc_fence_before();
  __syncthreads();
  if constexpr (CG == 2) cluster_sync();  // peer barriers initialised before any remote signal
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      // ===== TMA producer =====
      int stage = 0;
      uint32_t phase = 0;
      for (int unit = cid; unit < p.num_units; unit += ncl) {
        int tile, ks, hsel;
        decode_unit(p, unit, tile, ks, hsel);
        int b1, b2, m0, nt;
        decode_tile(p, tile, b1, b2, m0, nt);
        m0 += int(rank) * BM;
        // a half-width unit stages B rows [n0 + hsel BN/2 + rank BN/(2 CG), +BNL) (the box
        // is fixed; the MMA reads only the first BN/(2 CG) rows of each CTA's half)
        int n0 = nt * BN + (hsel < 0 ? int(rank) * BNL : hsel * (BN / 2) + int(rank) * (BNL / 2));
        // groups: the tile's group and its coordinates inside that group's maps
        int ga = 0, gb = 0;
        if (p.gdim == 1) {
          gb = (nt * BN) / p.gsize;
          n0 -= gb * p.gsize;
        } else if (p.gdim == 3) {
          ga = (m0 - int(rank) * BM) / p.gsize;
          m0 -= ga * p.gsize;
        }
        const int kb0 = ks * p.kb_per_split;
        const int kb1 = min(p.num_kb, kb0 + p.kb_per_split);
        for (int kb = kb0; kb < kb1; ++kb) {
          mbar_wait(&empty[stage], phase ^ 1);
          uint8_t* sa = smem + stage * STAGE;
          uint8_t* sb = sa + A_BYTES;
          int k0 = kb * BK;
          if (p.gdim == 2) {
            ga = gb = k0 / p.gsize;
            k0 -= ga * p.gsize;
          }
          const CUtensorMap* tmA = &tm.a[ga];
          const CUtensorMap* tmB = &tm.b[gb];
          if constexpr (CG == 1) {
            mbar_arrive_tx(&full[stage], STAGE);
            if (!p.a_mn) {
              tma_load(sa, tmA, &full[stage], k0, m0, b1, b2);
            } else {
#pragma unroll
              for (int i = 0; i < BM / 64; ++i) tma_load(sa + i * 8192, tmA, &full[stage], m0 + 64 * i, k0, b1, b2);
            }
            if (!p.b_mn) {
              tma_load(sb, tmB, &full[stage], k0, n0, b1, b2);
            } else {
#pragma unroll
              for (int i = 0; i < BNL / 64; ++i) tma_load(sb + i * 8192, tmB, &full[stage], n0 + 64 * i, k0, b1, b2);
            }
          } else {
            // both CTAs' bytes complete on the leader's barrier; only the leader arrives
            if (rank == 0) mbar_arrive_tx(&full[stage], 2 * STAGE);
            const uint32_t fb = mapa_shared(smem_u32(&full[stage]), 0);
            if (!p.a_mn) {
              tma_load_2sm(sa, tmA, fb, k0, m0, b1, b2);
            } else {
#pragma unroll
              for (int i = 0; i < BM / 64; ++i) tma_load_2sm(sa + i * 8192, tmA, fb, m0 + 64 * i, k0, b1, b2);
            }
            if (!p.b_mn) {
              tma_load_2sm(sb, tmB, fb, k0, n0, b1, b2);
            } else {
#pragma unroll
              for (int i = 0; i < BNL / 64; ++i) tma_load_2sm(sb + i * 8192, tmB, fb, n0 + 64 * i, k0, b1, b2);
            }
          }
          if (++stage == STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {
      // ===== MMA issuer (single thread; the pair leader for CG = 2) =====
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      // K-major SW128: rows of 128 B, 8-row groups 1024 B apart (SBO), K step = +32 B.
      // MN-major SW128: 64-element MN blocks 8 KB apart (LBO), 8-k groups 1024 B apart
      // (SBO), K step of 16 = +2048 B.
      const uint32_t a_lbo = p.a_mn ? 8192 : 16, b_lbo = p.b_mn ? 8192 : 16;
      const uint32_t a_kstep = p.a_mn ? 2048 : 32, b_kstep = p.b_mn ? 2048 : 32;
      for (int unit = cid; unit < p.num_units; unit += ncl) {
        int tile, ks, hsel;
        decode_unit(p, unit, tile, ks, hsel);
        const uint32_t id = hsel < 0 ? idesc : idesc_h;
        const int kb0 = ks * p.kb_per_split;
        const int kb1 = min(p.num_kb, kb0 + p.kb_per_split);
        mbar_wait(&tempty[acc], acc_phase ^ 1);
        tc_fence_after();
        const uint32_t tmem_d = tmem_base + uint32_t(acc * BN);
        for (int kb = kb0; kb < kb1; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          uint32_t sa = smem_u32(smem + stage * STAGE);
          uint32_t sb = sa + A_BYTES;
#pragma unroll
          for (int k = 0; k < BK / 16; ++k) {
            uint64_t ad = smem_desc(sa + k * a_kstep, a_lbo, 1024);
            uint64_t bd = smem_desc(sb + k * b_kstep, b_lbo, 1024);
            if constexpr (CG == 1) tc_mma(tmem_d, ad, bd, id, (kb > kb0 || k > 0) ? 1u : 0u);
            else tc_mma2(tmem_d, ad, bd, id, (kb > kb0 || k > 0) ? 1u : 0u);
          }
          if constexpr (CG == 1) tc_commit(&empty[stage]);
          else tc_commit2(&empty[stage], 3);
          if (++stage == STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
        if constexpr (CG == 1) tc_commit(&tfull[acc]);
        else tc_commit2(&tfull[acc], 3);
        if (++acc == 2) {
          acc = 0;
          acc_phase ^= 1;
        }
      }
    }
  } else {
    // ===== epilogue: TMEM -> registers (alpha, bias) -> swizzled smem -> TMA store =====
    const int q = warp & 3;        // TMEM lane quarter this warp may access
    const int ew = warp - 2;       // epilogue warp index
    const int half = ew >> 2;      // column group: chunks half, half + kGrp, ... of each tile
    constexpr int kGrp = EW / 4;
    constexpr int NBUF = staging_nbuf<F32OUT, EW, BNL>();
    uint8_t* wbuf = cstage + ew * NBUF * BUF;
    int nbuf = 0;
    int acc = 0;
    uint32_t acc_phase = 0;
    const int es = p.c_f32 ? 4 : 2;
    const uint32_t tempty_leader = CG == 2 ? mapa_shared(smem_u32(&tempty[0]), 0) : 0u;
    for (int unit = cid; unit < p.num_units; unit += ncl) {
      int tile, ks, hsel;
      decode_unit(p, unit, tile, ks, hsel);
      int b1, b2, m0, nt;
      decode_tile(p, tile, b1, b2, m0, nt);
      m0 += int(rank) * BM;
      const int n0 = nt * BN + (hsel < 0 ? 0 : hsel * (BN / 2));
      const int nchunks = (hsel < 0 ? BN : BN / 2) / 32;
      // output group and the tile's coordinates in that group's C map / bias
      int gc = 0, cn0 = n0, cm0 = m0;
      if (p.gdim == 1) {
        gc = (nt * BN) / p.gsize;
        cn0 = n0 - gc * p.gsize;
      } else if (p.gdim == 3) {
        gc = (m0 - int(rank) * BM) / p.gsize;
        cm0 = m0 - gc * p.gsize;
      }
      const void* bias = p.gdim == 1 ? p.bias_g[gc] : p.bias;
      const CUtensorMap* tmC = &tm.c[gc];
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const int row = m0 + q * 32 + lane;
      const bool row_ok = row < p.M;
      const int64_t cbase = int64_t(b1) * p.cbs1 + int64_t(b2) * p.cbs2 + int64_t(row) * p.ldc;
#pragma unroll 1
      for (int c = half; c < nchunks; c += kGrp) {
        uint32_t r[32];
        tmem_ld32(tmem_base + (uint32_t(q * 32) << 16) + uint32_t(acc * BN + c * 32), r);
        const int col0 = n0 + c * 32;
        const int ccol = cn0 + c * 32;  // column in the group's C map / bias
        if (col0 < p.N) {
          float v[32];
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]) * p.alpha;
          const bool full_chunk = col0 + 32 <= p.N;
          if (bias) {
            if (full_chunk && !p.bias_f32 && (reinterpret_cast<uintptr_t>(bias) & 15) == 0) {
              // 32 bias values as four 16-byte loads (the same address across the warp: one broadcast each)
              const uint4* bp = reinterpret_cast<const uint4*>(reinterpret_cast<const bf16*>(bias) + ccol);
#pragma unroll
              for (int j = 0; j < 4; ++j) {
                const uint4 u = __ldg(bp + j);
                const __nv_bfloat162* b2 = reinterpret_cast<const __nv_bfloat162*>(&u);
#pragma unroll
                for (int h = 0; h < 4; ++h) {
                  const float2 f = __bfloat1622float2(b2[h]);
                  v[8 * j + 2 * h] += f.x;
                  v[8 * j + 2 * h + 1] += f.y;
                }
              }
            } else {
#pragma unroll
              for (int i = 0; i < 32; ++i)
                if (full_chunk || col0 + i < p.N)
                  v[i] += p.bias_f32 ? reinterpret_cast<const float*>(bias)[ccol + i]
                                     : to_f(reinterpret_cast<const bf16*>(bias)[ccol + i]);
            }
          }
          if (p.tma_store) {
            if (!p.c_f32 && p.beta != 0.f && !p.reduce_add && row_ok) {  // bf16 accumulate: read the old row chunk
              const bf16* cp = reinterpret_cast<const bf16*>(p.C) + cbase + col0;
#pragma unroll
              for (int i = 0; i < 32; ++i)
                if (full_chunk || col0 + i < p.N) v[i] += p.beta * to_f(cp[i]);
            }
            if constexpr (!F32OUT) {
              if (p.epi == 2) {  // dU = bf16(dH) * gelu'(U): U's row chunk straight from global
                const bf16* up = p.aux + int64_t(row) * p.ldaux + col0;
                if (row_ok && full_chunk) {
                  uint4 u[4];
#pragma unroll
                  for (int j = 0; j < 4; ++j) u[j] = __ldg(reinterpret_cast<const uint4*>(up) + j);
                  const bf16* ub = reinterpret_cast<const bf16*>(u);
#pragma unroll
                  for (int i = 0; i < 32; ++i) v[i] = bf16_round(v[i]) * gelu_d(to_f(ub[i]));
                } else if (row_ok) {
#pragma unroll
                  for (int i = 0; i < 32; ++i)
                    if (col0 + i < p.N) v[i] = bf16_round(v[i]) * gelu_d(to_f(up[i]));
                }
              }
            }
            // stage 32 rows x 32 columns in swizzled smem, then one TMA store (or reduce-add)
            auto stage_store = [&](const float* vals, const CUtensorMap* map, bool radd) {
              uint8_t* buf = wbuf + nbuf * BUF;
              if (lane == 0) {  // the store that last used `buf` has read it
                if constexpr (NBUF == 1) bulk_wait_read0();
                else bulk_wait_read1();
              }
              __syncwarp();
              if constexpr (F32OUT) {
#pragma unroll
                for (int j = 0; j < 8; ++j) {  // 128 B row, SWIZZLE_128B
                  st_shared_v4(smem_u32(buf + lane * 128 + ((j ^ (lane & 7)) << 4)), __float_as_uint(vals[4 * j]),
                               __float_as_uint(vals[4 * j + 1]), __float_as_uint(vals[4 * j + 2]),
                               __float_as_uint(vals[4 * j + 3]));
                }
              } else {
#pragma unroll
                for (int j = 0; j < 4; ++j) {  // 64 B row, SWIZZLE_64B
                  uint4 o;
                  __nv_bfloat162* o2 = reinterpret_cast<__nv_bfloat162*>(&o);
#pragma unroll
                  for (int h = 0; h < 4; ++h)
                    o2[h] = __floats2bfloat162_rn(vals[8 * j + 2 * h], vals[8 * j + 2 * h + 1]);
                  st_shared_v4(smem_u32(buf + lane * 64 + ((j ^ ((lane >> 1) & 3)) << 4)), o.x, o.y, o.z, o.w);
                }
              }
              fence_async_smem();
              __syncwarp();
              if (lane == 0) {
                if (radd) tma_reduce_add(map, buf, ccol, cm0 + q * 32, b1, b2);
                else tma_store(map, buf, ccol, cm0 + q * 32, b1, b2);
                bulk_commit();
              }
              nbuf = (nbuf + 1) % NBUF;
            };
            stage_store(v, tmC, p.reduce_add);
            if constexpr (!F32OUT) {
              if (p.epi == 1) {  // second output: gelu of the stored (bf16) U
#pragma unroll
                for (int i = 0; i < 32; ++i) v[i] = gelu_f(bf16_round(v[i]));
                stage_store(v, &tm.c2, false);
              } else if (p.epi == 3) {  // second output: bf16(U) + residual, as the add kernel rounds
                const bf16* rp = p.aux + int64_t(row) * p.ldaux + col0;
                if (row_ok && full_chunk) {
                  uint4 u[4];
#pragma unroll
                  for (int j = 0; j < 4; ++j) u[j] = __ldg(reinterpret_cast<const uint4*>(rp) + j);
                  const bf16* rb = reinterpret_cast<const bf16*>(u);
#pragma unroll
                  for (int i = 0; i < 32; ++i) v[i] = bf16_round(v[i]) + to_f(rb[i]);
                } else {
#pragma unroll
                  for (int i = 0; i < 32; ++i)
                    v[i] = bf16_round(v[i]) + ((row_ok && col0 + i < p.N) ? to_f(rp[i]) : 0.f);
                }
                stage_store(v, &tm.c2, false);
              }
            }
          } else if (row_ok) {
            if (p.c_f32) {
              float* cp = reinterpret_cast<float*>(p.C) + cbase + col0;
#pragma unroll
              for (int i = 0; i < 32; ++i)
                if (col0 + i < p.N) cp[i] = v[i] + (p.beta != 0.f ? p.beta * cp[i] : 0.f);
            } else {
              bf16* cp = reinterpret_cast<bf16*>(p.C) + cbase + col0;
#pragma unroll
              for (int i = 0; i < 32; ++i)
                if (col0 + i < p.N) cp[i] = from_f<bf16>(v[i] + (p.beta != 0.f ? p.beta * to_f(cp[i]) : 0.f));
            }
          }
        }
        __syncwarp();
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        if constexpr (CG == 1) mbar_arrive(&tempty[acc]);
        else mbar_arrive_cluster(tempty_leader + uint32_t(acc * 8));
      }
      if (++acc == 2) {
        acc = 0;
        acc_phase ^= 1;
      }
    }
    if (lane == 0) bulk_wait_all();
    (void)es;
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  if constexpr (CG == 2) cluster_sync();  // no CTA leaves while its peer may still signal it
  if (warp == 1) {
    tc_fence_after();
    if constexpr (CG == 1)
      asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(TMEM_COLS));
    else
      asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(TMEM_COLS));
  }
}

PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
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

// 4-D map: (contiguous dim, row dim, batch1, batch2); box (box0, box1, 1, 1).
bool make_map(CUtensorMap* map, const void* ptr, int64_t ld, int64_t bs1, int64_t bs2, int64_t d0, int64_t d1, int nb1,
              int nb2, int box0, int box1, int es, CUtensorMapDataType dt, CUtensorMapSwizzle swz) {
  auto fn = encode_fn();
  if (!fn) return false;
  uintptr_t base = reinterpret_cast<uintptr_t>(ptr);
  if (base % 16 || (ld * es) % 16 || ld < d0) return false;
  if (nb1 > 1 && (bs1 * es) % 16) return false;
  if (nb2 > 1 && (bs2 * es) % 16) return false;
  cuuint64_t dims[4] = {cuuint64_t(d0), cuuint64_t(d1), cuuint64_t(nb1), cuuint64_t(nb2)};
  cuuint64_t s1 = ld * es;
  cuuint64_t s2 = nb1 > 1 ? bs1 * es : s1 * d1;
  cuuint64_t s3 = nb2 > 1 ? bs2 * es : s2 * nb1;
  s2 = (s2 + 15) / 16 * 16;
  s3 = (s3 + 15) / 16 * 16;
  cuuint64_t strides[3] = {s1, s2, s3};
  cuuint32_t box[4] = {cuuint32_t(box0), cuuint32_t(box1), 1, 1};
  cuuint32_t estr[4] = {1, 1, 1, 1};
  CUresult r = fn(map, dt, 4, reinterpret_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

bool make_operand_map(CUtensorMap* map, const GemmOperand& op, int64_t d0, int64_t d1, int nb1, int nb2, int box1) {
  return make_map(map, op.ptr, op.ld, op.bs1, op.bs2, d0, d1, nb1, nb2, 64, box1, 2, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16,
                  CU_TENSOR_MAP_SWIZZLE_128B);
}

int g_num_sms = 0;
int g_pair_slots = 0;  // co-resident CTA pairs (2-CTA clusters at one CTA per SM)
std::atomic<int64_t> g_launches{0};
std::atomic<int> g_mode{0};  // 0 auto, 1 single-CTA tiles only, 2 CTA pairs whenever legal
GemmConfig g_last{};

template <int BN, bool F32OUT, int EW = 8, int CG = 1>
void launch(const TmSet& tm, const TcParams& p, cudaStream_t st) {
  constexpr int STAGE = (BM + BN / CG) * BK * 2;
  const int smem = num_stages<BN / CG, F32OUT, EW>() * STAGE + 1024 + staging_bytes<F32OUT, EW, BN / CG>() + 1024;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(gemm_tc_kernel<BN, F32OUT, EW, CG>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    attr = true;
  }
  if constexpr (CG == 1) {
    int grid = p.num_units < g_num_sms ? p.num_units : g_num_sms;
    gemm_tc_kernel<BN, F32OUT, EW, 1><<<grid, num_threads<EW>(), smem, st>>>(tm, p);
  } else {
    const int pairs = p.num_units < g_pair_slots ? p.num_units : g_pair_slots;
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(2 * pairs);
    cfg.blockDim = dim3(num_threads<EW>());
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, gemm_tc_kernel<BN, F32OUT, EW, 2>, tm, p);
  }
  g_launches++;
}

// number of 2-CTA clusters of the pair kernel that fit on the device at once
int query_pair_slots() {
  constexpr int STAGE = (BM + 128) * BK * 2;
  const int smem = num_stages<128, false, 8>() * STAGE + 1024 + staging_bytes<false, 8, 128>() + 1024;
  cudaFuncSetAttribute(gemm_tc_kernel<256, false, 8, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(g_num_sms);
  cfg.blockDim = dim3(num_threads<8>());
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = 2;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, gemm_tc_kernel<256, false, 8, 2>, &cfg) != cudaSuccess || n <= 0) {
    cudaGetLastError();
    n = g_num_sms / 2;
  }
  return n;
}

}  // namespace

void gemm_tc_set_mode(int mode) { g_mode = mode; }  // bits 0-1 tile mode, bit 2 no tail split
GemmConfig gemm_tc_last_config() { return g_last; }

int64_t gemm_tc_launches() { return g_launches.load(); }

bool gemm_tc(const GemmArgs& g, cudaStream_t st) {
  if (g.in_dtype != BF16 || g.M <= 0 || g.N <= 0 || g.K <= 0) return false;
  if (g.K < 16 || g.N < 16) return false;  // tiny products: SIMT path (TMA zero-fills short M tiles)
  if (g_num_sms == 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_num_sms, cudaDevAttrMultiProcessorCount, dev);
    if (g_num_sms <= 0) return false;
    g_pair_slots = query_pair_slots();
  }
  // Tile width and split-K are chosen together (the Fig. 5 effect of small micro-ops,
  // P:L125): time ~ ceil(units / SMs) x per-unit time, with per-tile times from the
  // measured tcgen05 efficiency of each width (narrow tiles are smem-feed bound in
  // SS mode: 256 -> ~0.90, 128 -> ~0.65, 64 -> ~0.45 of peak).  Split-K needs an fp32,
  // contiguous, unbatched C (partials are TMA reduce-added).
  // CTA pairs (cta_group::2, 256 x bn units on two SMs) halve each SM's B feed: a pair
  // tile of width bn costs one SM what a single-CTA tile of width bn costs, at the
  // efficiency of a single-CTA tile twice as wide.
  // grouped products (horizontal fusion of micro-ops sharing an operand, see GemmArgs)
  const int G = g.groups > 1 ? g.groups : 1;
  int gsize = 0;
  if (G > 1) {
    if (G > kMaxGroups || g.gdim < 1 || g.gdim > 3 || g.nb1 * g.nb2 != 1 || g.epi) return false;
    if (g.beta != 0.f && g.beta != 1.f) return false;
    const int ext = g.gdim == 1 ? g.N : g.gdim == 2 ? g.K : g.M;
    if (ext % G) return false;
    gsize = ext / G;
    if (g.gdim == 2 && gsize % BK) return false;
  }
  const bool splitk_ok = g.c_dtype == F32 && g.nb1 * g.nb2 == 1 && g.ldc == g.N;
  const int num_kb_all = (g.K + BK - 1) / BK;
  const int mode = g_mode.load() & 3;
  // half-width tail units: measured +3-5 % for K <= 1024 products, -1-2 % for K = 4096
  // (the kernels run power-capped, so idle tail SMs are partly paid back in clock)
  const bool tail_split = (g_mode.load() & 4) == 0 && num_kb_all <= 32;
  int best_bn = 256, best_ks = 1, best_cg = 1;
  double best = 1e30;
  for (int cg : {1, 2}) {
    if (cg == 2 && (mode == 1 || g.M <= BM || g_pair_slots <= 0)) continue;
    // pairs pay a cluster launch/teardown and a cross-CTA handshake per unit: only
    // worth it for reductions of >= 8 k-blocks (measured: K = 64 products lose 25 %)
    if (cg == 2 && mode == 0 && num_kb_all < 8) continue;
    if (cg == 1 && mode == 2 && g.M > BM && g.N > 64 && g_pair_slots > 0) continue;
    const int slots = cg == 1 ? g_num_sms : g_pair_slots;
    if (G > 1 && g.gdim == 3 && gsize % (BM * cg)) continue;  // a tile never straddles M groups
    for (int bn : {256, 128, 64}) {
      if (bn > 64 && g.N <= bn / 2) continue;
      if (G > 1 && g.gdim == 1 && gsize % bn) continue;  // ... nor N groups
      if (cg == 2 && bn < 128) continue;
      const double eff = cg == 2 ? (bn == 256 ? 0.97 : 0.60) : (bn == 256 ? 0.90 : bn == 128 ? 0.65 : 0.45);
      int64_t tiles = int64_t((g.M + BM * cg - 1) / (BM * cg)) * ((g.N + bn - 1) / bn) * g.nb1 * g.nb2;
      // split-K: the widest split that still fills the machine when there are few tiles, plus
      // small splits (2..8) that even out a partial last wave (e.g. q/k/v dW: 48 pair tiles on
      // 74 slots -> 3 splits, two full waves); fp32, unbatched C only (partials reduce-added)
      int ks_cands[10], nks = 0;
      ks_cands[nks++] = 1;
      // (only when one wave of whole tiles leaves over a quarter of the machine idle: measured,
      // splitting 64 pair tiles on 74 slots (86 %) costs 13 % on the FFN dW products)
      if (splitk_ok && num_kb_all >= 16 && tiles * 4 < int64_t(slots) * 3) {
        if (tiles * 2 <= slots) ks_cands[nks++] = std::max(1, std::min(int(slots / tiles), num_kb_all / 8));
        for (int k2 = 2; k2 <= 8 && k2 <= num_kb_all / 8; ++k2) ks_cands[nks++] = k2;
      }
      for (int ci = 0; ci < nks; ++ci) {
      const int ks = ks_cands[ci];
      int64_t units = tiles * ks;
      double waves = double((units + slots - 1) / slots);
      // a tail wave at most half full runs as half-width units (decode_unit)
      if (tail_split && ks == 1 && bn / (2 * cg) >= 64 && tiles > slots && tiles % slots &&
          2 * (tiles % slots) <= slots)
        waves -= 0.5;
      // time in (tile-width x k-block) units, + the pair's fixed cost (~4 k-blocks of a
      // 256-wide tile, fitted to the BERT micro-op shapes), + the partial-tile reduce-adds
      const int kb_unit = (num_kb_all + ks - 1) / ks;
      double cost = waves * (bn / eff) * kb_unit + (cg == 2 ? 1024.0 : 0.0) + (ks > 1 ? 256.0 * ks : 0.0);
      if (cost < best - 1e-9) {
        best = cost;
        best_bn = bn;
        best_ks = ks;
        best_cg = cg;
      }
      }
    }
  }
  if (best > 1e29) return false;  // no legal tiling (grouped products)
  // one A / B / C map per group over that group's extents (a plain product: index 0)
  TmSet tm;
  std::memset(&tm, 0, sizeof(tm));
  const int Ma = g.gdim == 3 && G > 1 ? gsize : g.M;
  const int Nb = g.gdim == 1 && G > 1 ? gsize : g.N;
  const int Kg = g.gdim == 2 && G > 1 ? gsize : g.K;
  bool ok = true;
  for (int i = 0; i < G && ok; ++i) {
    const GemmOperand& A = (G > 1 && g.gdim != 1) ? g.ag[i] : g.a;
    const GemmOperand& Bo = (G > 1 && g.gdim != 3) ? g.bg[i] : g.b;
    if (A.mn_major != g.a.mn_major || Bo.mn_major != g.b.mn_major) return false;
    ok = A.mn_major ? make_operand_map(&tm.a[i], A, Ma, Kg, g.nb1, g.nb2, 64)
                    : make_operand_map(&tm.a[i], A, Kg, Ma, g.nb1, g.nb2, BM);
    ok = ok && (Bo.mn_major ? make_operand_map(&tm.b[i], Bo, Nb, Kg, g.nb1, g.nb2, 64)
                            : make_operand_map(&tm.b[i], Bo, Kg, Nb, g.nb1, g.nb2, best_bn / best_cg));
  }
  if (!ok) return false;
  TcParams p;
  p.gdim = G > 1 ? g.gdim : 0;
  p.gsize = gsize;
  for (int i = 0; i < kMaxGroups; ++i) p.bias_g[i] = (G > 1 && g.gdim == 1 && i < G) ? g.biasg[i] : g.bias;
  p.M = g.M;
  p.N = g.N;
  p.K = g.K;
  p.nb1 = g.nb1;
  p.nb2 = g.nb2;
  p.bm = BM * best_cg;
  p.tiles_m = (g.M + p.bm - 1) / p.bm;
  p.tiles_n = (g.N + best_bn - 1) / best_bn;
  p.num_tiles = p.tiles_m * p.tiles_n * g.nb1 * g.nb2;
  p.num_kb = (g.K + BK - 1) / BK;
  p.n_fastest = (int64_t(g.M) >= int64_t(g.N)) ? 1 : 0;
  p.a_mn = g.a.mn_major;
  p.b_mn = g.b.mn_major;
  p.C = g.c;
  p.ldc = g.ldc;
  p.cbs1 = g.cbs1;
  p.cbs2 = g.cbs2;
  p.c_f32 = g.c_dtype == F32;
  p.alpha = g.alpha;
  p.beta = g.beta;
  p.bias = g.bias;
  p.bias_f32 = g.bias_dtype == F32;
  // output: TMA store (bf16/f32) or TMA reduce-add (f32, beta == 1) when the view is aligned
  const int es = p.c_f32 ? 4 : 2;
  const int Nc = g.gdim == 1 && G > 1 ? gsize : g.N;
  const int Mc = g.gdim == 3 && G > 1 ? gsize : g.M;
  const int GC = (G > 1 && g.gdim != 2) ? G : 1;
  p.tma_store = 1;
  for (int i = 0; i < GC; ++i) {
    void* C = (G > 1 && g.gdim != 2) ? g.cg[i] : g.c;
    if (!make_map(&tm.c[i], C, g.ldc, g.cbs1, g.cbs2, Nc, Mc, g.nb1, g.nb2, 32, 32, es,
                  p.c_f32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16,
                  p.c_f32 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B))
      p.tma_store = 0;
  }
  if (g.beta != 0.f && g.beta != 1.f) p.tma_store = 0;
  if (G > 1 && !p.tma_store) return false;  // grouped outputs only through TMA stores
  // fused GELU epilogues need the bf16 TMA-store path (and no accumulation into C)
  p.epi = g.epi;
  p.aux = static_cast<const bf16*>(g.aux);
  p.ldaux = g.ldaux;
  tm.c2 = tm.c[0];
  if (g.epi) {
    if (!p.tma_store || p.c_f32 || g.beta != 0.f || !g.aux) return false;
    if (g.epi == 1 && !make_map(&tm.c2, g.aux, g.ldaux, 0, 0, g.N, g.M, 1, 1, 32, 32, 2,
                                CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, CU_TENSOR_MAP_SWIZZLE_64B))
      return false;
    if (g.epi == 2 && ((reinterpret_cast<uintptr_t>(g.aux) | uintptr_t(g.ldaux * 2)) & 15)) return false;
    if (g.epi == 3 && (((reinterpret_cast<uintptr_t>(g.aux) | uintptr_t(g.ldaux * 2)) & 15) || !g.aux2 ||
                       !make_map(&tm.c2, g.aux2, g.ldaux2, 0, 0, g.N, g.M, 1, 1, 32, 32, 2,
                                 CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, CU_TENSOR_MAP_SWIZZLE_64B)))
      return false;
    if (g.nb1 * g.nb2 != 1) return false;
  }
  // beta = 1 accumulates with a TMA reduce-add of the new tile (fp32, or bf16 gradients that
  // several backward ops add into: the old values never pass through registers)
  p.reduce_add = (p.tma_store && g.beta == 1.f) ? 1 : 0;
  // split-K for products with few output tiles and a long reduction (dW = dY^T X):
  // partial tiles are reduce-added in fp32 (the zero-init comes first when beta == 0)
  p.ksplit = 1;
  if (best_ks > 1 && p.tma_store && p.c_f32) {
    p.ksplit = best_ks;
    if (g.beta == 0.f) {
      if (G > 1 && g.gdim != 2)
        for (int i = 0; i < G; ++i) cudaMemsetAsync(g.cg[i], 0, size_t(Mc) * Nc * 4, st);
      else
        cudaMemsetAsync(g.c, 0, size_t(g.M) * g.N * 4, st);
    }
    p.reduce_add = 1;
  }
  p.kb_per_split = (p.num_kb + p.ksplit - 1) / p.ksplit;
  p.ksplit = (p.num_kb + p.kb_per_split - 1) / p.kb_per_split;
  p.num_units = p.num_tiles * p.ksplit;
  p.split_from = p.num_units;
  {
    const int slots = best_cg == 2 ? g_pair_slots : g_num_sms;
    const int tail = p.num_tiles % slots;
    if (tail_split && p.ksplit == 1 && best_bn / (2 * best_cg) >= 64 && p.num_tiles > slots && tail &&
        2 * tail <= slots) {
      p.split_from = p.num_tiles - tail;
      p.num_units = p.num_tiles + tail;
    }
  }
  g_last = GemmConfig{best_bn, best_cg, p.ksplit, p.num_units, g_num_sms, g_pair_slots, p.split_from};
  if (best_cg == 2) {
    if (p.c_f32) {
      if (best_bn == 256) launch<256, true, 8, 2>(tm, p, st);
      else launch<128, true, 8, 2>(tm, p, st);
    } else if (best_bn == 256) {
      if (p.epi) launch<256, false, 16, 2>(tm, p, st);
      else launch<256, false, 8, 2>(tm, p, st);
    } else {
      if (p.epi) launch<128, false, 16, 2>(tm, p, st);
      else launch<128, false, 8, 2>(tm, p, st);
    }
    return true;
  }
  if (p.c_f32) {
    switch (best_bn) {
      case 256: launch<256, true>(tm, p, st); break;
      case 128: launch<128, true>(tm, p, st); break;
      default: launch<64, true>(tm, p, st); break;
    }
  } else {
    switch (best_bn) {
      case 256:
        if (p.epi) launch<256, false, 16>(tm, p, st);
        else launch<256, false>(tm, p, st);
        break;
      case 128: launch<128, false>(tm, p, st); break;
      default: launch<64, false>(tm, p, st); break;
    }
  }
  return true;
}

static std::vector<GemmRecord>* g_sink = nullptr;
void gemm_records_enable(std::vector<GemmRecord>* sink) { g_sink = sink; }
std::vector<GemmRecord>* gemm_records_sink() { return g_sink; }

void gemm(const GemmArgs& g, cudaStream_t st) {
  GemmRecord rec{};
  if (g_sink) {
    cudaEventCreate(&rec.start);
    cudaEventCreate(&rec.stop);
    cudaEventRecord(rec.start, st);
  }
  rec.tc = gemm_tc(g, st) ? 1 : 0;
  if (!rec.tc && g.groups > 1) {
    // no tcgen05 tiling for the grouped product: run its groups as plain products
    const int G = g.groups;
    for (int i = 0; i < G; ++i) {
      GemmArgs s1 = g;
      s1.groups = 1;
      s1.gdim = 0;
      if (g.gdim == 1) {
        s1.N = g.N / G; s1.b = g.bg[i]; s1.c = g.cg[i]; s1.bias = g.biasg[i];
      } else if (g.gdim == 2) {
        s1.K = g.K / G; s1.a = g.ag[i]; s1.b = g.bg[i];
        if (i > 0) s1.beta = 1.f;
        if (i > 0) s1.bias = nullptr;
      } else {
        s1.M = g.M / G; s1.a = g.ag[i]; s1.c = g.cg[i];
      }
      std::vector<GemmRecord>* sink = g_sink;  // one record for the grouped product
      g_sink = nullptr;
      gemm(s1, st);
      g_sink = sink;
    }
  } else if (!rec.tc) {
    GemmArgs plain = g;
    plain.epi = 0;
    gemm_simt(plain, st);
    // the fused epilogue's effect, unfused: gelu of the stored U / dU = dH * gelu'(U) in place
    if (g.epi == 1) gelu_fwd(BF16, g.c, g.aux, int64_t(g.M) * g.N, st);
    if (g.epi == 2) gelu_bwd(BF16, g.c, g.aux, g.c, 0, int64_t(g.M) * g.N, st);
    if (g.epi == 3) add_fwd(BF16, g.c, g.aux, g.aux2, int64_t(g.M) * g.N, st);
  }
  if (g_sink) {
    cudaEventRecord(rec.stop, st);
    rec.flop = 2.0 * g.M * double(g.N) * g.K * g.nb1 * g.nb2;
    rec.M = g.M;
    rec.N = g.N;
    rec.K = g.K;
    rec.batch = g.nb1 * g.nb2;
    rec.flags = (g.a.mn_major ? 1 : 0) | (g.b.mn_major ? 2 : 0) | (g.c_dtype == F32 ? 4 : 0) | (g.beta != 0.f ? 8 : 0);
    g_sink->push_back(rec);
  }
}

}  // namespace tsk
