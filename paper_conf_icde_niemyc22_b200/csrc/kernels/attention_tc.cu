// Fused attention on the 5th-generation tensor cores (sm_100a), head dim 64, seq a multiple
// of 128 — the same arithmetic as attention.cu's kernels (dropout reading
// D-RNG), so the [b, a, s, s] score / probability / dropout tensors are never materialised
// (P:L119).  Three persistent warp-specialised kernels, each with TMA-fed operands in
// 128B-swizzled shared memory, tcgen05.mma issued by one thread and TMEM accumulators:
//   * fa5_fwd: online softmax over 64-key chunks (thresholded running max), O = P V, the row
//     log-sum-exp and the dropout keep bits (Philox on separate RNG warps);
//   * fa5_bwd_dq: dQ per 128-query tile (P rebuilt from S and the log-sum-exp, keep bits read);
//   * fa5_bwd_dkv: dK, dV per 128-key tile.
// Each kernel's layout and pipeline is described above it.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <mutex>

#include "common.cuh"
#include "kernels.h"
#include "tc_ptx.cuh"

namespace tsk {

namespace {

using namespace tc;

constexpr float kLog2e = 1.4426950408889634f;
constexpr float kLn2 = 0.6931471805599453f;

__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ void named_sync(int id, int n) { asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n)); }
__device__ __forceinline__ void sts128(uint32_t addr, uint32_t a, uint32_t b, uint32_t c, uint32_t d) {
  asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(addr), "r"(a), "r"(b), "r"(c), "r"(d) : "memory");
}
__device__ __forceinline__ uint32_t pk2(float lo, float hi) {
  __nv_bfloat162 h = __floats2bfloat162_rn(lo, hi);
  return *reinterpret_cast<uint32_t*>(&h);
}

struct Fa5P {
  int nb, heads, seq;
  int64_t ld;
  float sl2;          // alpha * log2(e)
  float p, keep_scale;
  uint32_t seed, step, thr;
  const uint32_t* step_ptr;  // live step counter (null: step)
  int64_t b0;
  void* c;
  float* lse;
  uint32_t* mask;
};

// ======================================================================= backward
// Shared by both backward kernels: 128 row threads (TMEM lane i = thread i), one control
// thread (TMA + tcgen05.mma).  P is rebuilt from S and the saved log-sum-exp, the keep
// bits come from the forward's mask (no Philox), D_q = dO_q . O_q.
struct Fa5B {
  int nb, heads, seq;
  int64_t ld;
  float sl2, alpha, keep_scale;
  int drop;
  const float* lse;
  const uint32_t* mask;
  float* D;             // [nb, heads, seq] row terms (dq5 writes, dkv5 reads)
  const bf16* o;        // forward output (dq5: D)
  const bf16* dout;
  void *dq, *dk, *dv;
  int acc_q, acc_k, acc_v;
};

// 16 compute warps (four per TMEM lane quarter, each owning 32 of a tile's 128 columns) + 1 control warp
constexpr int kBwdCW = 16;
constexpr uint32_t kIdN128 = (1u << 4) | (1u << 7) | (1u << 10) | (uint32_t(128 >> 3) << 17) | (uint32_t(128 >> 4) << 24);
constexpr uint32_t kIdN64MN = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | (uint32_t(64 >> 3) << 17) |
                              (uint32_t(128 >> 4) << 24);

// store 32 bf16 values of row i at keys [kl, kl+32) of a K-major SW128 operand (64-key blocks of 16 KB)
__device__ __forceinline__ void st_row32(uint32_t base, int i, int kl, const float* v) {
  const uint32_t blk = base + uint32_t(kl >> 6) * 16384u + uint32_t(i) * 128u;
#pragma unroll
  for (int q4 = 0; q4 < 4; ++q4) {
    const int chunk = ((kl & 63) >> 3) + q4;
    sts128(blk + (uint32_t(chunk ^ (i & 7)) << 4), pk2(v[8 * q4], v[8 * q4 + 1]), pk2(v[8 * q4 + 2], v[8 * q4 + 3]),
           pk2(v[8 * q4 + 4], v[8 * q4 + 5]), pk2(v[8 * q4 + 6], v[8 * q4 + 7]));
  }
}
__device__ __forceinline__ void tmem_ld32_nw(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
        "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
        "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }
// 32 columns of one row (scaled by sc, optionally added to the bf16 values already there)
__device__ __forceinline__ void store_row32(bf16* dst, const uint32_t (&r)[32], float sc, int acc) {
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    float f[8];
#pragma unroll
    for (int e = 0; e < 8; ++e) f[e] = __uint_as_float(r[8 * j + e]) * sc;
    uint4* pp = reinterpret_cast<uint4*>(dst + 8 * j);
    if (acc) {
      const uint4 old = *pp;
      const __nv_bfloat162* o2 = reinterpret_cast<const __nv_bfloat162*>(&old);
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float2 x = __bfloat1622float2(o2[e]);
        f[2 * e] += x.x;
        f[2 * e + 1] += x.y;
      }
    }
    *pp = make_uint4(pk2(f[0], f[1]), pk2(f[2], f[3]), pk2(f[4], f[5]), pk2(f[6], f[7]));
  }
}

// Both backward kernels put queries on the TMEM lanes of the score tiles (S = Q K^T and
// dP = dO V^T, M = 128 queries), so a thread's row constants — lse, D = dO.O and the keep
// word of its 32 keys — are per-thread scalars loaded once per tile.  16 compute warps
// (four per lane quarter, each owning 32 of the tile's 128 key columns) and one control
// thread.  The control thread issues the next tile's S, dP as soon as every compute warp has
// copied the current ones out of TMEM (s_free), and the bf16 operands the compute warps
// write (dS; P^T as well for dK/dV) are double-buffered in shared memory, so the tensor
// core works on tile t+1 while the compute warps are still on tile t.
//
// D[b, a, q] = dO_q . O_q over the 64 dims of head a (fp32 over the bf16 rows), the row term
// of both backward kernels; 8 lanes per (row, head), 16-byte loads, three shuffles.
__global__ void __launch_bounds__(256) attn_row_dot(const bf16* __restrict__ o, const bf16* __restrict__ g,
                                                    float* __restrict__ D, int64_t rows, int heads, int seq,
                                                    int64_t ld) {
  const int64_t t = int64_t(blockIdx.x) * 256 + threadIdx.x;
  const int64_t pair = t >> 3;  // (row, head)
  const int part = int(t & 7);
  const bool ok = pair < rows * heads;
  float d = 0.f;
  int64_t row = 0;
  int a = 0;
  if (ok) {
    row = pair / heads;
    a = int(pair - row * heads);
    const int64_t off = row * ld + a * 64 + part * 8;
    const uint4 x = *reinterpret_cast<const uint4*>(o + off), y = *reinterpret_cast<const uint4*>(g + off);
    const __nv_bfloat162* x2 = reinterpret_cast<const __nv_bfloat162*>(&x);
    const __nv_bfloat162* y2 = reinterpret_cast<const __nv_bfloat162*>(&y);
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const float2 u = __bfloat1622float2(x2[e]), w = __bfloat1622float2(y2[e]);
      d += u.x * w.x + u.y * w.y;
    }
  }
  d += __shfl_xor_sync(0xffffffffu, d, 1);
  d += __shfl_xor_sync(0xffffffffu, d, 2);
  d += __shfl_xor_sync(0xffffffffu, d, 4);
  if (ok && part == 0) {
    const int64_t b = row / seq, q = row - b * seq;
    D[(b * heads + a) * seq + q] = d;
  }
}

// dQ, persistent: a work item is 128 queries of one (sample, head); K and V stream through a
// 3-stage TMA ring one 128-key tile at a time (so the next item's loads run ahead), Q / dO
// are double-buffered per item, and dQ accumulates in one of two TMEM buffers so an item's
// epilogue overlaps the next item's products.  One TMA thread, one MMA thread, 16 compute
// warps.  D_q = dO_q . O_q comes from attn_row_dot (launched first).
// smem: Q 2 x 16K | dO 2 x 16K | K,V ring 3 x 32K | dS 2 x 32K | dS row partials 3 x 512 B | barriers
// TMEM: S 0..127, dP 128..255, dQ 256..319 / 320..383
constexpr int kDqStages = 3;
constexpr int kDqThreads = 32 * (kBwdCW + 2);
constexpr int kDqSmemQ = 0, kDqSmemG = 32768, kDqSmemKV = 65536, kDqSmemDS = kDqSmemKV + kDqStages * 32768;
constexpr int kDqSmemD = kDqSmemDS + 65536, kDqSmemBar = kDqSmemD + 1536;  // D: 3 x 128 row partials
constexpr int kDqSmem = kDqSmemBar + 256 + 1024;
__global__ void __launch_bounds__(kDqThreads, 1)
    fa5_bwd_dq(const __grid_constant__ CUtensorMap mQ, const __grid_constant__ CUtensorMap mdO,
               const __grid_constant__ CUtensorMap mK, const __grid_constant__ CUtensorMap mV, const Fa5B p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int S = p.seq, nkt = S / 128, nqt = S / 128;
  const int items = p.nb * p.heads * nqt;
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem + kDqSmemBar);
  uint64_t *qd_full = bar /*[2]*/, *qd_empty = bar + 2 /*[2]*/, *kv_full = bar + 4 /*[3]*/,
           *kv_empty = bar + 7 /*[3]*/, *s_full = bar + 10, *s_free = bar + 11, *ds_full = bar + 12 /*[2]*/,
           *ds_free = bar + 14 /*[2]*/, *dq_full = bar + 16 /*[2]*/, *dq_empty = bar + 18 /*[2]*/;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bar + 20);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  constexpr int kTma = kBwdCW, kMma = kBwdCW + 1;
  if (threadIdx.x == 0) {
    for (int i = 0; i < 2; ++i) {
      mbar_init(&qd_full[i], 1);
      mbar_init(&qd_empty[i], 1);
      mbar_init(&ds_full[i], 32 * kBwdCW);
      mbar_init(&ds_free[i], 1);
      mbar_init(&dq_full[i], 1);
      mbar_init(&dq_empty[i], 32 * kBwdCW);
    }
    for (int i = 0; i < kDqStages; ++i) {
      mbar_init(&kv_full[i], 1);
      mbar_init(&kv_empty[i], 1);
    }
    mbar_init(s_full, 1);
    mbar_init(s_free, 32 * kBwdCW);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kMma) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  if (warp == kTma) {
    if (lane == 0) {
      int it = 0, kc = 0;
      for (int item = blockIdx.x; item < items; item += gridDim.x, ++it) {
        const int qt = item % nqt, ah = item / nqt, a = ah % p.heads, b = ah / p.heads;
        const int row0 = b * S, buf = it & 1;
        if (it >= 2) mbar_wait(&qd_empty[buf], ((it >> 1) - 1) & 1);
        mbar_arrive_tx(&qd_full[buf], 32768u);
        tma_load(smem + kDqSmemQ + buf * 16384, &mQ, &qd_full[buf], a * 64, row0 + qt * 128, 0, 0);
        tma_load(smem + kDqSmemG + buf * 16384, &mdO, &qd_full[buf], a * 64, row0 + qt * 128, 0, 0);
        for (int kt = 0; kt < nkt; ++kt, ++kc) {
          const int st = kc % kDqStages;
          if (kc >= kDqStages) mbar_wait(&kv_empty[st], ((kc / kDqStages) - 1) & 1);
          mbar_arrive_tx(&kv_full[st], 32768u);
          tma_load(smem + kDqSmemKV + st * 32768, &mK, &kv_full[st], a * 64, row0 + kt * 128, 0, 0);
          tma_load(smem + kDqSmemKV + st * 32768 + 16384, &mV, &kv_full[st], a * 64, row0 + kt * 128, 0, 0);
        }
      }
    }
  } else if (warp == kMma) {
    if (lane == 0) {
      int it = 0, kc = 0;  // items, key tiles (running)
      uint32_t ns = 0;     // S / dP tiles issued
      for (int item = blockIdx.x; item < items; item += gridDim.x, ++it) {
        const int buf = it & 1, acc = it & 1;
        mbar_wait(&qd_full[buf], (it >> 1) & 1);
        const uint32_t q = smem_u32(smem + kDqSmemQ + buf * 16384), g = smem_u32(smem + kDqSmemG + buf * 16384);
        auto issue_dq = [&](int kcp, int first) {  // dQ += dS K of running tile kcp
          mbar_wait(&ds_full[kcp & 1], (kcp >> 1) & 1);
          tc_fence_after();
          const uint32_t dsb = smem_u32(smem + kDqSmemDS + (kcp & 1) * 32768);
          const uint32_t k = smem_u32(smem + kDqSmemKV + (kcp % kDqStages) * 32768);
          for (int kk = 0; kk < 128; kk += 16)
            tc_mma(tmem + 256 + uint32_t(acc * 64), smem_desc(dsb + (kk >> 6) * 16384 + ((kk & 63) >> 4) * 32, 16, 1024),
                   smem_desc(k + uint32_t(kk) * 128, 8192, 1024), kIdN64MN, (first && kk == 0) ? 0u : 1u);
          tc_commit(&ds_free[kcp & 1]);
          tc_commit(&kv_empty[kcp % kDqStages]);
        };
        for (int kt = 0; kt < nkt; ++kt, ++kc) {
          const int st = kc % kDqStages;
          mbar_wait(&kv_full[st], (kc / kDqStages) & 1);
          if (ns > 0) mbar_wait(s_free, (ns - 1) & 1);  // the previous S, dP are in registers
          tc_fence_after();
          const uint32_t k = smem_u32(smem + kDqSmemKV + st * 32768), v = k + 16384;
#pragma unroll
          for (int kk = 0; kk < 4; ++kk) {
            tc_mma(tmem, smem_desc(q + kk * 32, 16, 1024), smem_desc(k + kk * 32, 16, 1024), kIdN128, kk > 0 ? 1u : 0u);
            tc_mma(tmem + 128, smem_desc(g + kk * 32, 16, 1024), smem_desc(v + kk * 32, 16, 1024), kIdN128,
                   kk > 0 ? 1u : 0u);
          }
          tc_commit(s_full);
          ++ns;
          if (kt == nkt - 1) tc_commit(&qd_empty[buf]);  // every product reading Q, dO of this item issued
          if (kt > 0) {
            if (kt == 1 && it >= 2) mbar_wait(&dq_empty[acc], ((it >> 1) - 1) & 1);  // epilogue of item it-2 read dQ
            issue_dq(kc - 1, kt == 1);
          }
        }
        if (nkt == 1 && it >= 2) mbar_wait(&dq_empty[acc], ((it >> 1) - 1) & 1);
        issue_dq(kc - 1, nkt == 1);
        tc_commit(&dq_full[acc]);
      }
    }
  } else {
    const int qw = warp & 3, cg = warp >> 2;  // TMEM lane quarter, 32-column group
    const int i = qw * 32 + lane;
    const uint32_t trow = tmem + (uint32_t(qw * 32) << 16);
    int it = 0, kc = 0;
    // the row's D (attn_row_dot) and raw lse, loaded one item ahead (the loads complete while
    // the current item computes; nothing waits on them until the next item starts)
    // (row index of (sample, head) ah = b * heads + a: hr = ah * S + query)
    auto row_of = [&](int itm) {
      const int qt_ = itm % nqt, ah_ = itm / nqt;
      return int64_t(ah_) * S + qt_ * 128 + i;
    };
    auto item_consts = [&](int itm, float& D_, float& lse_) {
      const int64_t hr = row_of(itm);
      D_ = p.D[hr];
      lse_ = p.lse[hr];
    };
    float nD = 0.f, nlse = 0.f;
    // keep word of (item, key tile kt) for this row and 32-key group, loaded a tile ahead
    int64_t khr = 0;  // row of the item whose keep words load next
    auto keep_word = [&](int itm, int kt_) -> uint32_t {
      if (!p.drop) return ~0u;
      if (kt_ == 0) khr = row_of(itm);
      return p.mask[khr * (S / 32) + kt_ * 4 + cg];
    };
    uint32_t nbits = ~0u;
    if (int(blockIdx.x) < items) {
      item_consts(blockIdx.x, nD, nlse);
      nbits = keep_word(blockIdx.x, 0);
    }
    for (int item = blockIdx.x; item < items; item += gridDim.x, ++it) {
      const int qt = item % nqt, ah = item / nqt, a = ah % p.heads, b = ah / p.heads;
      const int q = qt * 128 + i;
      const float D = nD;
      const float l2 = nlse * kLog2e;
      float rsum = 0.f;  // this thread's share of sum_j dS_ij
      if (item + int(gridDim.x) < items) item_consts(item + gridDim.x, nD, nlse);
      for (int kt = 0; kt < nkt; ++kt, ++kc) {
        const uint32_t bits = nbits;
        if (kt + 1 < nkt) nbits = keep_word(item, kt + 1);
        else if (item + int(gridDim.x) < items) nbits = keep_word(item + gridDim.x, 0);
        mbar_wait(s_full, kc & 1);
        tc_fence_after();
        uint32_t rs[32], rp[32];
        tmem_ld32_nw(trow + uint32_t(cg * 32), rs);
        tmem_ld32_nw(trow + uint32_t(128 + cg * 32), rp);
        tmem_wait_ld();
        tc_fence_before();
        mbar_arrive(s_free);
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          const float pr = ex2(__uint_as_float(rs[j]) * p.sl2 - l2);
          const float dp = ((bits >> j) & 1u) ? __uint_as_float(rp[j]) * p.keep_scale : 0.f;
          const float ds = pr * (dp - D);
          rsum += ds;
          rs[j] = __float_as_uint(ds);
        }
        if (kc >= 2) mbar_wait(&ds_free[kc & 1], ((kc >> 1) - 1) & 1);  // the dQ product of tile kc-2 read it
        st_row32(smem_u32(smem + kDqSmemDS + (kc & 1) * 32768), i, cg * 32, reinterpret_cast<const float*>(rs));
        fence_async_smem();
        tc_fence_before();
        mbar_arrive(&ds_full[kc & 1]);
      }
      // the dK/dV kernel's row term: D_i = sum_j P_ij dP_ij over the P rebuilt here, i.e. the
      // dO . O of attn_row_dot plus sum_j dS_ij (dO . O carries the bf16 rounding of O; with
      // the consistent D, dS has zero row sums and the key-bias gradient its analytic zero).
      // Four column groups per row: fixed-order sum through shared memory (deterministic).
      {
        float* red = reinterpret_cast<float*>(smem + kDqSmemD);
        if (cg > 0) red[(cg - 1) * 128 + i] = rsum;
        named_sync(1, 32 * kBwdCW);
        if (cg == 0) {
          const int64_t hr = (int64_t(b) * p.heads + a) * S + q;
          p.D[hr] = D + (((rsum + red[i]) + red[128 + i]) + red[256 + i]);
        }
        named_sync(1, 32 * kBwdCW);  // the slots are rewritten by the next item
      }
      mbar_wait(&dq_full[it & 1], (it >> 1) & 1);
      tc_fence_after();
      if (cg < 2) {
        uint32_t r0[32];
        tmem_ld32(trow + 256u + uint32_t((it & 1) * 64 + cg * 32), r0);
        if (p.dq)
          store_row32(static_cast<bf16*>(p.dq) + (int64_t(b) * S + q) * p.ld + a * 64 + cg * 32, r0, p.alpha, p.acc_q);
      }
      tc_fence_before();
      mbar_arrive(&dq_empty[it & 1]);
    }
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  if (warp == kMma) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512));
  }
}

// dK, dV, persistent: a work item is 128 keys of one (sample, head); K and V are
// double-buffered per item, Q and dO stream through a 3-stage TMA ring one 128-query tile at
// a time, and dK / dV accumulate in one of two TMEM buffer pairs so an item's epilogue
// overlaps the next item's products.  P_d (dropped, scaled P) and dS are written query-major
// ([query][key] rows, SW128) — the MN-major layout of the A operands P_d^T and dS^T of
// dV += P_d^T dO and dK += dS^T Q.  One TMA thread, one MMA thread, 16 compute warps.
// smem: K,V 2 x 32K | Q,dO ring 3 x 32K | P_d 32K | dS 32K | barriers
// TMEM: S 0..127, dP 128..255 (lanes = queries); dV, dK 256..383 / 384..511 (lanes = keys)
constexpr int kKvStages = 3;
constexpr int kKvThreads = 32 * (kBwdCW + 2);
constexpr int kKvSmemKV = 0, kKvSmemQG = 65536, kKvSmemPd = kKvSmemQG + kKvStages * 32768;
constexpr int kKvSmemDS = kKvSmemPd + 32768, kKvSmemBar = kKvSmemDS + 32768;
constexpr int kKvSmem = kKvSmemBar + 256 + 1024;
__global__ void __launch_bounds__(kKvThreads, 1)
    fa5_bwd_dkv(const __grid_constant__ CUtensorMap mQ, const __grid_constant__ CUtensorMap mdO,
                const __grid_constant__ CUtensorMap mK, const __grid_constant__ CUtensorMap mV, const Fa5B p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int S = p.seq, nqt = S / 128, nkt = S / 128;
  const int items = p.nb * p.heads * nkt;
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem + kKvSmemBar);
  uint64_t *kv_full = bar /*[2]*/, *kv_empty = bar + 2 /*[2]*/, *qd_full = bar + 4 /*[3]*/, *qd_empty = bar + 7 /*[3]*/,
           *s_full = bar + 10, *s_free = bar + 11, *ps_full = bar + 12, *ps_free = bar + 13,
           *acc_full = bar + 14 /*[2]*/, *acc_empty = bar + 16 /*[2]*/;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bar + 18);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  constexpr int kTma = kBwdCW, kMma = kBwdCW + 1;
  if (threadIdx.x == 0) {
    for (int i = 0; i < 2; ++i) {
      mbar_init(&kv_full[i], 1);
      mbar_init(&kv_empty[i], 1);
      mbar_init(&acc_full[i], 1);
      mbar_init(&acc_empty[i], 32 * kBwdCW);
    }
    for (int i = 0; i < kKvStages; ++i) {
      mbar_init(&qd_full[i], 1);
      mbar_init(&qd_empty[i], 1);
    }
    mbar_init(s_full, 1);
    mbar_init(s_free, 32 * kBwdCW);
    mbar_init(ps_full, 32 * kBwdCW);
    mbar_init(ps_free, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kMma) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  if (warp == kTma) {
    if (lane == 0) {
      int it = 0, qc = 0;
      for (int item = blockIdx.x; item < items; item += gridDim.x, ++it) {
        const int kt = item % nkt, ah = item / nkt, a = ah % p.heads, b = ah / p.heads;
        const int row0 = b * S, kb = it & 1;
        if (it >= 2) mbar_wait(&kv_empty[kb], ((it >> 1) - 1) & 1);
        mbar_arrive_tx(&kv_full[kb], 32768u);
        tma_load(smem + kKvSmemKV + kb * 32768, &mK, &kv_full[kb], a * 64, row0 + kt * 128, 0, 0);
        tma_load(smem + kKvSmemKV + kb * 32768 + 16384, &mV, &kv_full[kb], a * 64, row0 + kt * 128, 0, 0);
        for (int t = 0; t < nqt; ++t, ++qc) {
          const int st = qc % kKvStages;
          if (qc >= kKvStages) mbar_wait(&qd_empty[st], ((qc / kKvStages) - 1) & 1);
          mbar_arrive_tx(&qd_full[st], 32768u);
          tma_load(smem + kKvSmemQG + st * 32768, &mQ, &qd_full[st], a * 64, row0 + t * 128, 0, 0);
          tma_load(smem + kKvSmemQG + st * 32768 + 16384, &mdO, &qd_full[st], a * 64, row0 + t * 128, 0, 0);
        }
      }
    }
  } else if (warp == kMma) {
    if (lane == 0) {
      // dV += P_d^T dO_t, dK += dS^T Q_t: A MN-major (keys contiguous, 64-key blocks 16 KB apart,
      // K step of 16 queries = 2 KB), B = dO / Q tile rows (MN-major)
      constexpr uint32_t idAcc = kIdN64MN | (1u << 15);
      const uint32_t pd = smem_u32(smem + kKvSmemPd), ds = smem_u32(smem + kKvSmemDS);
      int it = 0, qc = 0;
      for (int item = blockIdx.x; item < items; item += gridDim.x, ++it) {
        const int kb = it & 1, ab = it & 1;
        mbar_wait(&kv_full[kb], (it >> 1) & 1);
        const uint32_t k = smem_u32(smem + kKvSmemKV + kb * 32768), v = k + 16384;
        auto issue_acc = [&](int qcp, int first) {
          mbar_wait(ps_full, qcp & 1);
          tc_fence_after();
          const uint32_t q = smem_u32(smem + kKvSmemQG + (qcp % kKvStages) * 32768), g = q + 16384;
          for (int kq = 0; kq < 128; kq += 16) {
            const uint32_t acc = (first && kq == 0) ? 0u : 1u;
            tc_mma(tmem + 256 + uint32_t(ab * 128), smem_desc(pd + uint32_t(kq) * 128, 16384, 1024),
                   smem_desc(g + uint32_t(kq) * 128, 8192, 1024), idAcc, acc);
            tc_mma(tmem + 320 + uint32_t(ab * 128), smem_desc(ds + uint32_t(kq) * 128, 16384, 1024),
                   smem_desc(q + uint32_t(kq) * 128, 8192, 1024), idAcc, acc);
          }
          tc_commit(ps_free);
          tc_commit(&qd_empty[qcp % kKvStages]);
        };
        for (int t = 0; t < nqt; ++t, ++qc) {
          const int st = qc % kKvStages;
          mbar_wait(&qd_full[st], (qc / kKvStages) & 1);
          if (qc > 0) mbar_wait(s_free, (qc - 1) & 1);  // the previous S, dP are in registers
          tc_fence_after();
          const uint32_t q = smem_u32(smem + kKvSmemQG + st * 32768), g = q + 16384;
          // S = Q_t K^T, dP = dO_t V^T (M = 128 queries, N = 128 keys)
#pragma unroll
          for (int kk = 0; kk < 4; ++kk) {
            tc_mma(tmem, smem_desc(q + kk * 32, 16, 1024), smem_desc(k + kk * 32, 16, 1024), kIdN128, kk > 0 ? 1u : 0u);
            tc_mma(tmem + 128, smem_desc(g + kk * 32, 16, 1024), smem_desc(v + kk * 32, 16, 1024), kIdN128,
                   kk > 0 ? 1u : 0u);
          }
          tc_commit(s_full);
          if (t == nqt - 1) tc_commit(&kv_empty[kb]);  // every product reading K, V of this item issued
          if (t > 0) {
            if (t == 1 && it >= 2) mbar_wait(&acc_empty[ab], ((it >> 1) - 1) & 1);
            issue_acc(qc - 1, t == 1);
          }
        }
        if (nqt == 1 && it >= 2) mbar_wait(&acc_empty[ab], ((it >> 1) - 1) & 1);
        issue_acc(qc - 1, nqt == 1);
        tc_commit(&acc_full[ab]);
      }
    }
  } else {
    const int qw = warp & 3, cg = warp >> 2;  // TMEM lane quarter, 32-key group
    const int i = qw * 32 + lane;
    const uint32_t trow = tmem + (uint32_t(qw * 32) << 16);
    const uint32_t pd = smem_u32(smem + kKvSmemPd), ds = smem_u32(smem + kKvSmemDS);
    int it = 0, qc = 0;
    // row constants (raw lse, D, keep word) of query tile t of a work item
    // (row index of (sample, head) ah = b * heads + a: hr = ah * S + query; one division per
    // work item — the per-tile integer divisions were a twentieth of this kernel's stall samples)
    int nah = 0, nkt_ = 0;  // (sample, head) and key tile of the item whose constants load next
    auto row_consts = [&](int itm, int t, float& lse_, float& D_, uint32_t& bits_) {
      if (t == 0) {
        nkt_ = itm % nkt;
        nah = itm / nkt;
      }
      const int kt_ = nkt_;
      const int64_t hr = int64_t(nah) * S + t * 128 + i;
      lse_ = p.lse[hr];
      D_ = p.D[hr];
      bits_ = p.drop ? p.mask[hr * (S / 32) + kt_ * 4 + cg] : ~0u;
    };
    float nlse = 0.f, nD = 0.f;
    uint32_t nbits = ~0u;
    if (int(blockIdx.x) < items) row_consts(blockIdx.x, 0, nlse, nD, nbits);
    for (int item = blockIdx.x; item < items; item += gridDim.x, ++it) {
      const int kt = item % nkt, ah = item / nkt, a = ah % p.heads, b = ah / p.heads;
      for (int t = 0; t < nqt; ++t, ++qc) {
        // this tile's constants were loaded one tile (or, for t = 0, one item) ahead; the
        // raw lse is scaled only now, so no instruction waits on a load issued just before
        const float l2 = nlse * kLog2e, D = nD;
        const uint32_t bits = nbits;
        if (t + 1 < nqt) row_consts(item, t + 1, nlse, nD, nbits);
        else if (item + int(gridDim.x) < items) row_consts(item + gridDim.x, 0, nlse, nD, nbits);
        mbar_wait(s_full, qc & 1);
        tc_fence_after();
        uint32_t rs[32], rp[32];
        tmem_ld32_nw(trow + uint32_t(cg * 32), rs);
        tmem_ld32_nw(trow + uint32_t(128 + cg * 32), rp);
        tmem_wait_ld();
        tc_fence_before();
        mbar_arrive(s_free);
        // in place: rp <- P_d, rs <- dS (fp32 bits)
#pragma unroll
        for (int j = 0; j < 32; ++j) {
          // one select: km = keep_scale or 0, then dP_d = dP km and P_d = P km (a dropped dP of
          // either sign gives +-0, and +-0 - D = -D: the same values as selecting each)
          const float km = ((bits >> j) & 1u) ? p.keep_scale : 0.f;
          const float pr = ex2(__uint_as_float(rs[j]) * p.sl2 - l2);
          const float dp = __uint_as_float(rp[j]) * km;
          rp[j] = __float_as_uint(pr * km);
          rs[j] = __float_as_uint(pr * (dp - D));
        }
        if (qc > 0) mbar_wait(ps_free, (qc - 1) & 1);  // the previous tile's dV, dK products read P_d / dS
        st_row32(pd, i, cg * 32, reinterpret_cast<const float*>(rp));
        st_row32(ds, i, cg * 32, reinterpret_cast<const float*>(rs));
        fence_async_smem();
        tc_fence_before();
        mbar_arrive(ps_full);
      }
      mbar_wait(&acc_full[it & 1], (it >> 1) & 1);
      tc_fence_after();
      // accumulator lanes are keys: group 0/1 store dV columns 0-31 / 32-63, group 2/3 dK
      const int key = kt * 128 + i;
      const int64_t off = (int64_t(b) * S + key) * p.ld + a * 64 + (cg & 1) * 32;
      uint32_t r0[32];
      tmem_ld32(trow + 256u + uint32_t((it & 1) * 128 + cg * 32), r0);
      tc_fence_before();
      mbar_arrive(&acc_empty[it & 1]);
      if (cg < 2) {
        if (p.dv) store_row32(static_cast<bf16*>(p.dv) + off, r0, 1.f, p.acc_v);
      } else {
        if (p.dk) store_row32(static_cast<bf16*>(p.dk) + off, r0, p.alpha, p.acc_k);
      }
    }
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  if (warp == kMma) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512));
  }
}

// ======================================================================= forward
// Persistent, warp-specialised forward.  A work item is a pair of 128-query tiles of one
// (sample, head); K and V stream through a 4-stage TMA ring in 64-key chunks, so any seq
// that is a multiple of 128 works.  Per tile t of the pair, two softmax warpgroups (key
// halves h = 0, 1 of every chunk) run an online softmax over the chunks: S_t = Q_t K_j^T
// lands in one of two TMEM buffers (lanes = queries), so the tensor core computes chunk j+1
// while the softmax warps work on chunk j; a thread owns one row and 32 keys of the chunk,
// copies them to registers and releases the buffer at once.  The chunk max is exchanged
// between the halves through shared memory; the running max only moves when it grows by
// more than 8 (log2 units) — then the warp rescales its half of the O_t rows in TMEM after
// the previous P V product has landed — otherwise the stale max is kept (exponentials
// stay <= 2^8; exact after the final 1/l).  P (dropout applied) goes to shared memory in the
// K-major SW128 layout and O_t += P V_j runs on the tensor cores.  The keep bits (one Philox
// call per eight keys of a row, reading D-RNG) come from eight RNG warps — thread = (tile, row),
// both key halves of a chunk, up to two chunks ahead through a double-buffered shared-memory
// slot — which also write the mask output: the Philox integer work (about 40 % of the forward's
// instructions) runs on warps of its own, interleaved with the softmax warps' MUFU / FMA work by
// the schedulers, and setmaxnreg moves the RNG and control warps' unused registers to the
// softmax warps (157 -> 146 us per BERT-Large layer at p = 0.1, the same bits and values).  One
// thread issues TMA and one thread per query tile issues that tile's tcgen05.mma products (S of
// chunk j+1 before P V of chunk j), so neither tile's next S waits for the other tile's P
// (146 -> 142.5 us); the next item's Q and the next chunks' K / V load while the current item
// computes.
//   TMEM: S_0 [0,64) [64,128)  S_1 [128,192) [192,256)  O_0 [256,320)  O_1 [320,384)
//   smem: Q 2 x 16K | K,V ring 4 x 16K | P 2 x 16K | barriers, row exchange
constexpr int kFwdSoftWarps = 16;  // (tile t, key half h, lane quarter): warp = 8t + 4h + quarter
constexpr int kFwdRngWarps = 8;    // (tile t, lane quarter): warp = kFwdSoftWarps + 4t + quarter
constexpr int kFwdTma = kFwdSoftWarps + kFwdRngWarps, kFwdMma = kFwdTma + 1;
constexpr int kFwdThreads = 32 * (kFwdSoftWarps + kFwdRngWarps + 4);  // + TMA, 2 x MMA, one idle warp
// setmaxnreg split of the 896 x 72 registers allocated at launch (softmax warps hold a 32-key
// S slice, the exchange and the P tile addressing; RNG threads eight Philox states)
constexpr uint32_t kFwdRegSoft = 80, kFwdRegRng = 64, kFwdRegCtl = 56;
constexpr int kFwdKC = 64;  // keys per chunk
constexpr int kFwdStages = 4;
constexpr int kFwdSmemQ = 0, kFwdSmemKV = 32768, kFwdSmemP = kFwdSmemKV + kFwdStages * 16384;
constexpr int kFwdSmemBar = kFwdSmemP + 32768;
constexpr int kFwdSmemBits = kFwdSmemBar + 512 + 6144;  // keep words [t][chunk parity][128 rows][2]
constexpr int kFwdSmem = kFwdSmemBits + 4096 + 1024;  // barriers | exchange: maxima [t][h][2][128], sums [t][h][128] | bits | align
constexpr float kRescaleThr = 8.f;

__device__ __forceinline__ void tmem_st32(uint32_t taddr, const uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
      "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
      "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]), "r"(r[17]), "r"(r[18]),
      "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]),
      "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31]));
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void sts32(uint32_t addr, float v) {
  asm volatile("st.shared.f32 [%0], %1;" ::"r"(addr), "f"(v) : "memory");
}
__device__ __forceinline__ float lds32(uint32_t addr) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(addr) : "memory");
  return v;
}

__global__ void __launch_bounds__(kFwdThreads, 1)
    fa5_fwd(const __grid_constant__ CUtensorMap mQ, const __grid_constant__ CUtensorMap mK,
            const __grid_constant__ CUtensorMap mV, const Fa5P p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem + kFwdSmemBar);
  uint64_t *q_full = bar, *q_empty = bar + 2, *kv_full = bar + 3, *kv_empty = bar + 3 + kFwdStages;
  // per tile: s_full[2], s_free[2], p_full, p_free, o_full, o_free
  uint64_t* tb = bar + 3 + 2 * kFwdStages;
  auto s_full = [&](int t, int b) { return tb + 8 * t + b; };
  auto s_free = [&](int t, int b) { return tb + 8 * t + 2 + b; };
  auto p_full = [&](int t) { return tb + 8 * t + 4; };
  auto p_free = [&](int t) { return tb + 8 * t + 5; };
  auto o_full = [&](int t) { return tb + 8 * t + 6; };
  auto o_free = [&](int t) { return tb + 8 * t + 7; };
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tb + 16);
  // keep words produced by the RNG warps: b_full[t][k] (RNG threads of tile t), b_free[t][k]
  // (its softmax threads), k = chunk parity
  auto b_full = [&](int t, int k) { return bar + 40 + 2 * t + k; };
  auto b_free = [&](int t, int k) { return bar + 44 + 2 * t + k; };
  const uint32_t xch = smem_u32(smem + kFwdSmemBar + 512);  // floats: maxima [t][h][2][128] | sums [t][h][128]
  const uint32_t bits_smem = smem_u32(smem + kFwdSmemBits);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int S = p.seq, nqt = S / 128, npair = (nqt + 1) / 2, nkc = S / kFwdKC;
  const int items = p.nb * p.heads * npair;
  const uint32_t step = p.step_ptr ? *p.step_ptr : p.step;
  if (threadIdx.x == 0) {
    mbar_init(&q_full[0], 1);
    mbar_init(&q_full[1], 1);
    mbar_init(q_empty, 2);  // one arrival per tile's MMA thread
    for (int s = 0; s < kFwdStages; ++s) {
      mbar_init(&kv_full[s], 1);
      mbar_init(&kv_empty[s], 2);
    }
    for (int t = 0; t < 2; ++t) {
      for (int b = 0; b < 2; ++b) {
        mbar_init(s_full(t, b), 1);
        mbar_init(s_free(t, b), 256);
      }
      mbar_init(p_full(t), 256);
      mbar_init(p_free(t), 1);
      mbar_init(o_full(t), 1);
      mbar_init(o_free(t), 256);
      for (int kk = 0; kk < 2; ++kk) {
        mbar_init(b_full(t, kk), 128);
        mbar_init(b_free(t, kk), 256);
      }
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kFwdMma) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(512));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp >= kFwdTma) {
   asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(kFwdRegCtl));
   if (warp == kFwdTma) {
    if (lane == 0) {
      int it = 0, kc = 0;  // items done by this CTA, K/V chunks loaded
      for (int item = blockIdx.x; item < items; item += gridDim.x, ++it) {
        const int pair = item % npair, ah = item / npair, a = ah % p.heads, b = ah / p.heads;
        const int row0 = b * S;
        const int nt = min(2, nqt - 2 * pair);
        if (it > 0) mbar_wait(q_empty, (it - 1) & 1);
        for (int t = 0; t < nt; ++t) {
          mbar_arrive_tx(&q_full[t], 16384u);
          tma_load(smem + kFwdSmemQ + t * 16384, &mQ, &q_full[t], a * 64, row0 + (2 * pair + t) * 128, 0, 0);
        }
        for (int j = 0; j < nkc; ++j, ++kc) {
          const int s = kc % kFwdStages;
          if (kc >= kFwdStages) mbar_wait(&kv_empty[s], ((kc / kFwdStages) - 1) & 1);
          uint8_t* st = smem + kFwdSmemKV + s * 16384;
          mbar_arrive_tx(&kv_full[s], 16384u);
          tma_load(st, &mK, &kv_full[s], a * 64, row0 + j * kFwdKC, 0, 0);
          tma_load(st + 8192, &mV, &kv_full[s], a * 64, row0 + j * kFwdKC, 0, 0);
        }
      }
    }
  } else if ((warp == kFwdMma || warp == kFwdMma + 1) && lane == 0) {
      // one tcgen05.mma-issuing thread per query tile, so neither tile's products wait behind
      // the other tile's P (the K/V stage and Q buffers are released by both: counts of 2)
      const int t = warp - kFwdMma;
      constexpr uint32_t idS = (1u << 4) | (1u << 7) | (1u << 10) | (uint32_t(kFwdKC >> 3) << 17) |
                               (uint32_t(128 >> 4) << 24);
      constexpr uint32_t idO = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 16) | (uint32_t(64 >> 3) << 17) |
                               (uint32_t(128 >> 4) << 24);
      int kc = 0;
      uint32_t cs = 0;   // S chunks issued (running: buffer cs & 1)
      uint32_t np = 0;   // p_full completions consumed
      uint32_t nit = 0;  // items (q_full / o_free phases)
      auto issue_s = [&](int st) {
        const uint32_t c = cs++, bsel = c & 1;
        if (c >= 2) mbar_wait(s_free(t, bsel), ((c >> 1) - 1) & 1);  // the buffer's previous chunk is read
        tc_fence_after();
        const uint32_t q = smem_u32(smem + kFwdSmemQ + t * 16384), k = smem_u32(smem + kFwdSmemKV + st * 16384);
#pragma unroll
        for (int kk = 0; kk < 4; ++kk)
          tc_mma(tmem + uint32_t(t * 128 + bsel * 64), smem_desc(q + kk * 32, 16, 1024),
                 smem_desc(k + kk * 32, 16, 1024), idS, kk > 0 ? 1u : 0u);
        tc_commit(s_full(t, bsel));
      };
      for (int item = blockIdx.x; item < items; item += gridDim.x) {
        const int pair = item % npair;
        const int nt = min(2, nqt - 2 * pair);
        if (t >= nt) {  // single-tile item: keep the shared stage / Q barriers' arrival counts
          for (int j = 0; j < nkc; ++j, ++kc) {
            const int st = kc % kFwdStages;
            mbar_wait(&kv_full[st], (kc / kFwdStages) & 1);
            if (j == 0) mbar_arrive(q_empty);
            mbar_arrive(&kv_empty[st]);
          }
          continue;
        }
        {
          const int st = kc % kFwdStages;
          mbar_wait(&kv_full[st], (kc / kFwdStages) & 1);
          mbar_wait(&q_full[t], nit & 1);
          issue_s(st);
        }
        for (int j = 0; j < nkc; ++j, ++kc) {
          const int st = kc % kFwdStages;
          const uint32_t v = smem_u32(smem + kFwdSmemKV + st * 16384 + 8192);
          const bool more = j + 1 < nkc;
          if (more) {  // chunk j+1 into the other S buffer
            mbar_wait(&kv_full[(kc + 1) % kFwdStages], ((kc + 1) / kFwdStages) & 1);
            issue_s((kc + 1) % kFwdStages);
          }
          mbar_wait(p_full(t), np & 1);
          ++np;
          if (j == 0 && nit > 0) mbar_wait(o_free(t), (nit - 1) & 1);
          tc_fence_after();
          const uint32_t pb = smem_u32(smem + kFwdSmemP + t * 16384);
#pragma unroll
          for (int kk = 0; kk < kFwdKC; kk += 16)
            tc_mma(tmem + 256 + uint32_t(t * 64), smem_desc(pb + (kk >> 4) * 32, 16, 1024),
                   smem_desc(v + uint32_t(kk) * 128, 8192, 1024), idO, (j > 0 || kk > 0) ? 1u : 0u);
          tc_commit(p_free(t));
          if (!more) tc_commit(o_full(t));
          tc_commit(&kv_empty[st]);
        }
        ++nit;
        tc_commit(q_empty);
      }
   }
  } else if (warp >= kFwdSoftWarps) {
    // ===== RNG warps: tile t, row i — the keep bits of each 64-key chunk (both halves), up to two
    // chunks ahead of the softmax warps, and the mask output
    asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(kFwdRegRng));
    const int t = (warp - kFwdSoftWarps) >> 2, i = ((warp - kFwdSoftWarps) & 3) * 32 + lane;
    uint32_t cb = 0;  // chunks produced (this tile)
    for (int item = blockIdx.x; item < items; item += gridDim.x) {
      const int pair = item % npair, ah = item / npair, a = ah % p.heads, b = ah / p.heads;
      const int nt = min(2, nqt - 2 * pair);
      if (t >= nt) continue;
      const int q = (2 * pair + t) * 128 + i;
      const uint64_t erow = ((uint64_t(p.b0 + b) * p.heads + a) * uint64_t(S) + uint64_t(q)) * uint64_t(S);
      uint32_t* mrow = p.mask ? p.mask + ((int64_t(b) * p.heads + a) * S + q) * (S / 32) : nullptr;
      for (int j = 0; j < nkc; ++j, ++cb) {
        const int key = j * kFwdKC;
        uint32_t w0 = 0xFFFFFFFFu, w1 = 0xFFFFFFFFu;
        if (p.p > 0.f) {
          // one Philox call per eight keys of the row (D-RNG); erow + key is a multiple of 64,
          // so the eight counters share the high word
          const uint64_t cnt0 = (erow + uint64_t(key)) >> 3;
          w0 = 0u;
          w1 = 0u;
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const uint4 x0 = philox4x32_10(uint32_t(cnt0) + uint32_t(u), uint32_t(cnt0 >> 32), step, 0u, p.seed,
                                           kPhiloxKey1);
            w0 |= keep_bits8(x0, p.thr) << (8 * u);
          }
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            const uint4 x1 = philox4x32_10(uint32_t(cnt0) + uint32_t(4 + u), uint32_t(cnt0 >> 32), step, 0u, p.seed,
                                           kPhiloxKey1);
            w1 |= keep_bits8(x1, p.thr) << (8 * u);
          }
        }
        if (mrow) *reinterpret_cast<uint2*>(mrow + (key >> 5)) = make_uint2(w0, w1);
        if (!(p.p > 0.f)) continue;  // no dropout: the softmax warps need no bits
        const int kb = cb & 1;
        if (cb >= 2) mbar_wait(b_free(t, kb), ((cb >> 1) - 1) & 1);
        asm volatile("st.shared.v2.b32 [%0], {%1, %2};" ::"r"(bits_smem + uint32_t(((t * 2 + kb) * 128 + i) * 8)),
                     "r"(w0), "r"(w1)
                     : "memory");
        mbar_arrive(b_full(t, kb));
      }
    }
  } else {
    // ===== softmax warps: tile t, key half h (32 keys of each chunk), row i
    asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(kFwdRegSoft));
    const int t = warp >> 3, h = (warp >> 2) & 1, qq = warp & 3;
    const int i = qq * 32 + lane;
    const uint32_t srow = tmem + (uint32_t(qq * 32) << 16) + uint32_t(t * 128 + 32 * h);
    const uint32_t orow = tmem + (uint32_t(qq * 32) << 16) + 256u + uint32_t(t * 64 + 32 * h);
    const uint32_t pbuf = smem_u32(smem + kFwdSmemP + t * 16384);
    const uint32_t xm = xch + uint32_t(t * 2) * 1024u;         // [h][2][128] floats
    const uint32_t xl = xch + 4096u + uint32_t(t) * 1024u;     // [h][128] floats
    const int bar_id = 1 + t;                                  // named barrier of the tile's 256 threads
    uint32_t cs = 0, npw = 0, nit = 0;  // S chunks read, P tiles written, items (this tile)
    for (int item = blockIdx.x; item < items; item += gridDim.x) {
      const int pair = item % npair, ah = item / npair, a = ah % p.heads, b = ah / p.heads;
      const int nt = min(2, nqt - 2 * pair);
      if (t >= nt) continue;
      const int q = (2 * pair + t) * 128 + i;
      float mrun = -INFINITY, l = 0.f;
      for (int j = 0; j < nkc; ++j, ++cs) {
        const uint32_t bsel = cs & 1;
        mbar_wait(s_full(t, bsel), (cs >> 1) & 1);
        tc_fence_after();
        uint32_t r[32];
        tmem_ld32(srow + bsel * 64u, r);
        tc_fence_before();
        mbar_arrive(s_free(t, bsel));
        // chunk max over the 64 keys (this half's 32, exchanged with the other half)
        float m = -INFINITY;
#pragma unroll
        for (int jj = 0; jj < 32; ++jj) m = fmaxf(m, __uint_as_float(r[jj]));
        sts32(xm + uint32_t((h * 2 + (j & 1)) * 128 + i) * 4u, m);
        named_sync(bar_id, 256);
        m = fmaxf(m, lds32(xm + uint32_t(((h ^ 1) * 2 + (j & 1)) * 128 + i) * 4u)) * p.sl2;
        // the running max moves when it grows by more than kRescaleThr; the O_t row rescale is a
        // warp-collective TMEM access, so the warp takes it when any of its rows needs it
        const bool grow = m > mrun + kRescaleThr;
        const float f = grow ? ex2(mrun - m) : 1.f;
        l *= f;
        if (j > 0 && __any_sync(0xffffffffu, grow)) {
          mbar_wait(p_free(t), (npw - 1) & 1);  // P V of chunk j-1 has landed in O_t
          tc_fence_after();
          uint32_t o[32];
          tmem_ld32(orow, o);
#pragma unroll
          for (int jj = 0; jj < 32; ++jj) o[jj] = __float_as_uint(__uint_as_float(o[jj]) * f);
          tmem_st32(orow, o);
          tmem_wait_st();
        }
        if (grow) mrun = m;
        // P = 2^(S alpha log2e - mrun) with the keep bits, bf16 into the K-major P tile
        float* v = reinterpret_cast<float*>(r);
#pragma unroll
        for (int jj = 0; jj < 32; ++jj) {
          v[jj] = ex2(fmaf(v[jj], p.sl2, -mrun));
          l += v[jj];
        }
        // this half's 32 keep bits from the RNG warp of the row (D-RNG; bit jj = key j kFwdKC + 32 h + jj)
        if (p.p > 0.f) {
          const int kb = cs & 1;
          mbar_wait(b_full(t, kb), (cs >> 1) & 1);
          uint32_t bits;
          asm volatile("ld.shared.b32 %0, [%1];"
                       : "=r"(bits)
                       : "r"(bits_smem + uint32_t(((t * 2 + kb) * 128 + i) * 8 + h * 4))
                       : "memory");
          mbar_arrive(b_free(t, kb));
#pragma unroll
          for (int jj = 0; jj < 32; ++jj)
            if (!((bits >> jj) & 1u)) v[jj] = 0.f;
        }
        if (npw > 0) mbar_wait(p_free(t), (npw - 1) & 1);  // the previous P V has read the P tile
        st_row32(pbuf, i, 32 * h, v);
        ++npw;
        fence_async_smem();
        tc_fence_before();
        mbar_arrive(p_full(t));
      }
      // epilogue: O_t row / l (keep_scale folded in), C and the log-sum-exp
      sts32(xl + uint32_t(h * 128 + i) * 4u, l);
      named_sync(bar_id, 256);
      const float lt = l + lds32(xl + uint32_t((h ^ 1) * 128 + i) * 4u);
      mbar_wait(o_full(t), nit & 1);
      ++nit;
      tc_fence_after();
      uint32_t o[32];
      tmem_ld32(orow, o);
      tc_fence_before();
      mbar_arrive(o_free(t));
      const float inv = p.keep_scale / lt;
      if (p.c) {
        bf16* crow = static_cast<bf16*>(p.c) + (int64_t(b) * S + q) * p.ld + a * 64 + 32 * h;
#pragma unroll
        for (int jj = 0; jj < 4; ++jj) {
          uint4 ov;
          ov.x = pk2(__uint_as_float(o[8 * jj]) * inv, __uint_as_float(o[8 * jj + 1]) * inv);
          ov.y = pk2(__uint_as_float(o[8 * jj + 2]) * inv, __uint_as_float(o[8 * jj + 3]) * inv);
          ov.z = pk2(__uint_as_float(o[8 * jj + 4]) * inv, __uint_as_float(o[8 * jj + 5]) * inv);
          ov.w = pk2(__uint_as_float(o[8 * jj + 6]) * inv, __uint_as_float(o[8 * jj + 7]) * inv);
          *reinterpret_cast<uint4*>(crow + 8 * jj) = ov;
        }
      }
      if (h == 0 && p.lse) p.lse[(int64_t(b) * p.heads + a) * S + q] = (mrun + log2f(lt)) * kLn2;
      named_sync(bar_id, 256);  // the sum slots are reused by the next item
    }
  }
  __syncwarp();
  tc_fence_before();
  __syncthreads();
  if (warp == kFwdMma) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512));
  }
}

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

// [rows, ld] bf16 as a 4-D map (ld, rows, 1, 1) — tma_load issues the 4-D form —
// box (64 columns, box_rows rows), 128-byte swizzle
bool map2(CUtensorMap* m, const void* ptr, int64_t ld, int64_t rows, int box_rows) {
  auto fn = encode();
  if (!fn || reinterpret_cast<uintptr_t>(ptr) % 16 || (ld * 2) % 16) return false;
  cuuint64_t dims[4] = {cuuint64_t(ld), cuuint64_t(rows), 1, 1};
  cuuint64_t str[3] = {cuuint64_t(ld * 2), cuuint64_t(ld * 2 * rows), cuuint64_t(ld * 2 * rows)};
  cuuint32_t box[4] = {64, cuuint32_t(box_rows), 1, 1};
  cuuint32_t es[4] = {1, 1, 1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(ptr), dims, str, box, es,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

}  // namespace

bool attention_fwd_tc5(const AttnArgs& A, cudaStream_t st) {
  // (a recompute replay may regenerate only C, only lse or only the keep bits: each output
  // is written when its pointer is set)
  if (A.dtype != BF16 || A.d != 64 || A.seq % 128 || A.nb < 1 || (!A.c && !A.lse && !A.mask)) return false;
  const int64_t rows = int64_t(A.nb) * A.seq;
  CUtensorMap mq, mk, mv;
  if (!map2(&mq, A.q, A.ld, rows, 128) || !map2(&mk, A.k, A.ld, rows, kFwdKC) ||
      !map2(&mv, A.v, A.ld, rows, kFwdKC))
    return false;
  Fa5P p;
  p.nb = A.nb;
  p.heads = A.heads;
  p.seq = A.seq;
  p.ld = A.ld;
  p.sl2 = A.alpha * kLog2e;
  p.p = A.p;
  p.keep_scale = A.p > 0.f ? 1.f / (1.f - A.p) : 1.f;
  p.seed = A.seed;
  p.step = A.step;
  p.step_ptr = A.step_ptr;
  p.thr = A.thr;
  p.b0 = A.b0;
  p.c = A.c;
  p.lse = A.lse;
  p.mask = A.mask;
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaFuncSetAttribute(fa5_fwd, cudaFuncAttributeMaxDynamicSharedMemorySize, kFwdSmem);
  }
  const int items = A.nb * A.heads * ((A.seq / 128 + 1) / 2);
  fa5_fwd<<<items < sms ? items : sms, kFwdThreads, kFwdSmem, st>>>(mq, mk, mv, p);
  return true;
}

bool attention_bwd_tc5(const AttnArgs& A, cudaStream_t st) {
  if (A.dtype != BF16 || A.d != 64 || A.seq % 128 || A.seq > 512 || A.nb < 1 || !A.c || !A.lse || !A.mask ||
      !A.dc || !A.ws)
    return false;
  const int64_t rows = int64_t(A.nb) * A.seq;
  CUtensorMap mq, mg, mk, mv;
  if (!map2(&mq, A.q, A.ld, rows, 128) || !map2(&mg, A.dc, A.ld, rows, 128) || !map2(&mk, A.k, A.ld, rows, 128) ||
      !map2(&mv, A.v, A.ld, rows, 128))
    return false;
  Fa5B p;
  p.heads = A.heads;
  p.seq = A.seq;
  p.ld = A.ld;
  p.sl2 = A.alpha * kLog2e;
  p.alpha = A.alpha;
  p.keep_scale = A.p > 0.f ? 1.f / (1.f - A.p) : 1.f;
  p.drop = A.p > 0.f;
  p.lse = A.lse;
  p.mask = A.mask;
  p.D = A.ws;
  p.o = static_cast<const bf16*>(A.c);
  p.dout = static_cast<const bf16*>(A.dc);
  p.dq = A.dq;
  p.dk = A.dk;
  p.dv = A.dv;
  p.acc_q = A.acc_q;
  p.acc_k = A.acc_k;
  p.acc_v = A.acc_v;
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaFuncSetAttribute(fa5_bwd_dq, cudaFuncAttributeMaxDynamicSharedMemorySize, kDqSmem);
    cudaFuncSetAttribute(fa5_bwd_dkv, cudaFuncAttributeMaxDynamicSharedMemorySize, kKvSmem);
  }
  p.nb = A.nb;
  {
    const int64_t threads = rows * A.heads * 8;
    attn_row_dot<<<int((threads + 255) / 256), 256, 0, st>>>(static_cast<const bf16*>(A.c),
                                                           static_cast<const bf16*>(A.dc), A.ws, rows, A.heads,
                                                           A.seq, A.ld);
  }
  const int items_q = A.nb * A.heads * (A.seq / 128);
  fa5_bwd_dq<<<items_q < sms ? items_q : sms, kDqThreads, kDqSmem, st>>>(mq, mg, mk, mv, p);
  fa5_bwd_dkv<<<items_q < sms ? items_q : sms, kKvThreads, kKvSmem, st>>>(mq, mg, mk, mv, p);
  return true;
}

}  // namespace tsk
