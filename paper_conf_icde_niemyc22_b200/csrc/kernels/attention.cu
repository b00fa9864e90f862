// Fused attention micro-op: C = dropout(softmax(alpha Q_h K_h^T)) V_h
// per (sample, head), with the row log-sum-exp kept for the backward — none of the
// [b,a,s,s] scores / probabilities / dropped probabilities touches HBM (they are
// 3 x 268 MB per BERT-Large layer in the unfused graph, Table II's largest class).
// The dropout mask is the unfused op's (Philox4x32-10 on the element index of the
// [b,a,s,s] probabilities, DESIGN.md D-RNG), so both graphs compute the same function.
//
// Two implementations of the same arithmetic:
//  * tensor-core (bf16, head dim 64, seq % 64 == 0): FlashAttention-2 structure on
//    mma.sync m16n8k16 (fp32 accumulate) with ldmatrix from XOR-swizzled shared tiles
//    filled by cp.async (double-buffered).  Forward: CTA = 64 queries x one head, online
//    softmax over 64-key blocks.  Backward: a query-major kernel (dQ, and the row term
//    D_i = dO_i . O_i it stores for the second kernel) and a key-major kernel (dK, dV),
//    both recomputing P from Q, K and the saved log-sum-exp — no atomics, so results do
//    not depend on scheduling.
//  * CUDA cores (fp32 graphs, other shapes): one block per query (or key) row, fp64
//    accumulation for fp32 data.
#include "common.cuh"
#include "kernels.h"

namespace tsk {

namespace {

constexpr float kLog2e = 1.4426950408889634f;
constexpr float kLn2 = 0.6931471805599453f;

__device__ __forceinline__ uint32_t philox_one(uint64_t e, uint32_t seed, uint32_t step) {
  return philox_u16(e, seed, step);  // the element's 16-bit draw (D-RNG)
}

// Keep decisions of one 8-column n-tile of an mma.sync accumulator, for this thread's
// (row r, cols 2t, 2t+1) and (row r + 8, same cols): one Philox call covers the eight keys
// of a row (D-RNG), so lanes t = 0 / 1 of the quad draw rows r / r + 8 and every lane takes
// word t (its two keys' halves) of both by shuffles.
// e0 = element index of (row r of lane 0's quad, column 0 of the n-tile); S = row stride.
__device__ __forceinline__ void quad_keep(uint64_t e0, uint64_t S, uint32_t seed, uint32_t step, uint32_t thr,
                                          bool (&k)[4]) {
  const int lane = threadIdx.x & 31, t = lane & 3;
  const uint64_t c = (e0 + uint64_t(t & 1) * 8ull * S) >> 3;
  const uint4 r = philox4x32_10(uint32_t(c), uint32_t(c >> 32), step, 0u, seed, kPhiloxKey1);
  const int src0 = lane & ~3, src1 = src0 | 1;
  const uint32_t a0 = __shfl_sync(0xffffffffu, r.x, src0), a1 = __shfl_sync(0xffffffffu, r.y, src0);
  const uint32_t a2 = __shfl_sync(0xffffffffu, r.z, src0), a3 = __shfl_sync(0xffffffffu, r.w, src0);
  const uint32_t b0 = __shfl_sync(0xffffffffu, r.x, src1), b1 = __shfl_sync(0xffffffffu, r.y, src1);
  const uint32_t b2 = __shfl_sync(0xffffffffu, r.z, src1), b3 = __shfl_sync(0xffffffffu, r.w, src1);
  const uint32_t wa = t == 0 ? a0 : t == 1 ? a1 : t == 2 ? a2 : a3;
  const uint32_t wb = t == 0 ? b0 : t == 1 ? b1 : t == 2 ? b2 : b3;
  k[0] = (wa & 0xFFFFu) >= thr;
  k[1] = (wa >> 16) >= thr;
  k[2] = (wb & 0xFFFFu) >= thr;
  k[3] = (wb >> 16) >= thr;
}
__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

__device__ __forceinline__ bool mask_bit(const uint32_t* mrow, int key) { return (mrow[key >> 5] >> (key & 31)) & 1u; }

// ============================================================ CUDA-core version
template <class T>
struct AccOf {
  typedef float type;
};
template <>
struct AccOf<float> {
  typedef double type;
};

// one block per (query row i, head a, sample b); dynamic smem: seq accumulators
template <class T>
__global__ void attn_fwd_simt(AttnArgs A) {
  typedef typename AccOf<T>::type Acc;
  extern __shared__ __align__(16) uint8_t sm_raw[];
  Acc* s = reinterpret_cast<Acc*>(sm_raw);
  __shared__ Acc red[32];
  const int i = blockIdx.x, a = blockIdx.y, b = blockIdx.z;
  const int S = A.seq, d = A.d;
  const T* q = static_cast<const T*>(A.q) + (int64_t(b) * S + i) * A.ld + a * d;
  const T* k = static_cast<const T*>(A.k) + int64_t(b) * S * A.ld + a * d;
  const T* v = static_cast<const T*>(A.v) + int64_t(b) * S * A.ld + a * d;
  for (int j = threadIdx.x; j < S; j += blockDim.x) {
    Acc acc = 0;
    for (int t = 0; t < d; ++t) acc += Acc(to_f(q[t])) * Acc(to_f(k[int64_t(j) * A.ld + t]));
    s[j] = Acc(A.alpha) * acc;
  }
  __syncthreads();
  Acc m = -1e300;
  for (int j = threadIdx.x; j < S; j += blockDim.x) m = s[j] > m ? s[j] : m;
  for (int o = 16; o > 0; o >>= 1) {
    Acc x = __shfl_xor_sync(0xffffffffu, m, o);
    m = x > m ? x : m;
  }
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = m;
  __syncthreads();
  m = red[0];
  for (int w = 1; w < int(blockDim.x >> 5); ++w) m = red[w] > m ? red[w] : m;
  __syncthreads();
  Acc l = 0;
  for (int j = threadIdx.x; j < S; j += blockDim.x) l += exp(s[j] - m);
  for (int o = 16; o > 0; o >>= 1) l += __shfl_xor_sync(0xffffffffu, l, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = l;
  __syncthreads();
  l = 0;
  for (int w = 0; w < int(blockDim.x >> 5); ++w) l += red[w];
  const Acc lse = m + log(l);
  const uint64_t e0 = ((uint64_t(A.b0 + b) * A.heads + a) * S + i) * uint64_t(S);
  const Acc scale = A.p > 0.f ? Acc(1) / (Acc(1) - Acc(A.p)) : Acc(1);
  const uint32_t step = A.step_ptr ? *A.step_ptr : A.step;
  __syncthreads();
  for (int j = threadIdx.x; j < S; j += blockDim.x) {
    Acc pj = exp(s[j] - lse);
    if (A.p > 0.f) pj = philox_one(e0 + j, A.seed, step) >= A.thr ? pj * scale : Acc(0);
    s[j] = pj;
  }
  __syncthreads();
  if (A.c) {
    T* c = static_cast<T*>(A.c) + (int64_t(b) * S + i) * A.ld + a * d;
    for (int t = threadIdx.x; t < d; t += blockDim.x) {
      Acc acc = 0;
      for (int j = 0; j < S; ++j) acc += s[j] * Acc(to_f(v[int64_t(j) * A.ld + t]));
      c[t] = from_f<T>(float(acc));
    }
  }
  if (A.lse && threadIdx.x == 0) A.lse[(int64_t(b) * A.heads + a) * S + i] = float(lse);
  if (A.mask) {
    const int nw = (S + 31) / 32;
    uint32_t* mrow = A.mask + ((int64_t(b) * A.heads + a) * S + i) * nw;
    for (int w = threadIdx.x; w < nw; w += blockDim.x) {
      uint32_t bits = 0;
      for (int j = 0; j < 32 && 32 * w + j < S; ++j)
        if (A.p <= 0.f || philox_one(e0 + 32 * w + j, A.seed, step) >= A.thr) bits |= 1u << j;
      mrow[w] = bits;
    }
  }
}

// query-major backward: dQ_i and D_i = sum_j P_ij dP_ij (= dO_i . O_i), stored to ws
template <class T>
__global__ void attn_bwd_q_simt(AttnArgs A) {
  typedef typename AccOf<T>::type Acc;
  extern __shared__ __align__(16) uint8_t sm_raw[];
  Acc* P = reinterpret_cast<Acc*>(sm_raw);
  Acc* dP = P + A.seq;
  __shared__ Acc red[32];
  const int i = blockIdx.x, a = blockIdx.y, b = blockIdx.z;
  const int S = A.seq, d = A.d;
  const int64_t row = (int64_t(b) * S + i) * A.ld + a * d;
  const T* q = static_cast<const T*>(A.q) + row;
  const T* dc = static_cast<const T*>(A.dc) + row;
  const T* k = static_cast<const T*>(A.k) + int64_t(b) * S * A.ld + a * d;
  const T* v = static_cast<const T*>(A.v) + int64_t(b) * S * A.ld + a * d;
  const Acc lse = A.lse[(int64_t(b) * A.heads + a) * S + i];
  const uint32_t* mrow = A.mask + ((int64_t(b) * A.heads + a) * S + i) * ((S + 31) / 32);
  const Acc scale = A.p > 0.f ? Acc(1) / (Acc(1) - Acc(A.p)) : Acc(1);
  Acc part = 0;
  for (int j = threadIdx.x; j < S; j += blockDim.x) {
    Acc sq = 0, dd = 0;
    for (int t = 0; t < d; ++t) {
      sq += Acc(to_f(q[t])) * Acc(to_f(k[int64_t(j) * A.ld + t]));
      dd += Acc(to_f(dc[t])) * Acc(to_f(v[int64_t(j) * A.ld + t]));
    }
    const Acc pj = exp(Acc(A.alpha) * sq - lse);
    Acc dpj = dd;
    if (A.p > 0.f) dpj = mask_bit(mrow, j) ? dpj * scale : Acc(0);
    P[j] = pj;
    dP[j] = dpj;
    part += pj * dpj;
  }
  for (int o = 16; o > 0; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = part;
  __syncthreads();
  Acc D = 0;
  for (int w = 0; w < int(blockDim.x >> 5); ++w) D += red[w];
  if (threadIdx.x == 0) A.ws[(int64_t(b) * A.heads + a) * S + i] = float(D);
  for (int j = threadIdx.x; j < S; j += blockDim.x) P[j] = P[j] * (dP[j] - D);  // dS
  __syncthreads();
  if (A.dq) {
    T* dq = static_cast<T*>(A.dq) + row;
    for (int t = threadIdx.x; t < d; t += blockDim.x) {
      Acc acc = 0;
      for (int j = 0; j < S; ++j) acc += P[j] * Acc(to_f(k[int64_t(j) * A.ld + t]));
      float r = float(Acc(A.alpha) * acc);
      if (A.acc_q) r += to_f(dq[t]);
      dq[t] = from_f<T>(r);
    }
  }
}

// key-major backward: dK_j, dV_j (reads D from ws)
template <class T>
__global__ void attn_bwd_kv_simt(AttnArgs A) {
  typedef typename AccOf<T>::type Acc;
  extern __shared__ __align__(16) uint8_t sm_raw[];
  Acc* dS = reinterpret_cast<Acc*>(sm_raw);
  Acc* Pd = dS + A.seq;
  const int j = blockIdx.x, a = blockIdx.y, b = blockIdx.z;
  const int S = A.seq, d = A.d;
  const int64_t row = (int64_t(b) * S + j) * A.ld + a * d;
  const T* kj = static_cast<const T*>(A.k) + row;
  const T* vj = static_cast<const T*>(A.v) + row;
  const T* q = static_cast<const T*>(A.q) + int64_t(b) * S * A.ld + a * d;
  const T* dc = static_cast<const T*>(A.dc) + int64_t(b) * S * A.ld + a * d;
  const float* lse = A.lse + (int64_t(b) * A.heads + a) * S;
  const float* D = A.ws + (int64_t(b) * A.heads + a) * S;
  const Acc scale = A.p > 0.f ? Acc(1) / (Acc(1) - Acc(A.p)) : Acc(1);
  for (int i = threadIdx.x; i < S; i += blockDim.x) {
    Acc sq = 0, dd = 0;
    for (int t = 0; t < d; ++t) {
      sq += Acc(to_f(q[int64_t(i) * A.ld + t])) * Acc(to_f(kj[t]));
      dd += Acc(to_f(dc[int64_t(i) * A.ld + t])) * Acc(to_f(vj[t]));
    }
    const Acc pij = exp(Acc(A.alpha) * sq - Acc(lse[i]));
    bool keep = true;
    if (A.p > 0.f) keep = mask_bit(A.mask + ((int64_t(b) * A.heads + a) * S + i) * ((S + 31) / 32), j);
    const Acc dpij = keep ? dd * scale : Acc(0);
    Pd[i] = keep ? pij * scale : Acc(0);
    dS[i] = pij * (dpij - Acc(D[i]));
  }
  __syncthreads();
  T* dk = static_cast<T*>(A.dk) + row;
  T* dv = static_cast<T*>(A.dv) + row;
  for (int t = threadIdx.x; t < d; t += blockDim.x) {
    Acc ak = 0, av = 0;
    for (int i = 0; i < S; ++i) {
      ak += dS[i] * Acc(to_f(q[int64_t(i) * A.ld + t]));
      av += Pd[i] * Acc(to_f(dc[int64_t(i) * A.ld + t]));
    }
    if (A.dk) {
      float r = float(Acc(A.alpha) * ak);
      if (A.acc_k) r += to_f(dk[t]);
      dk[t] = from_f<T>(r);
    }
    if (A.dv) {
      float r = float(av);
      if (A.acc_v) r += to_f(dv[t]);
      dv[t] = from_f<T>(r);
    }
  }
}

// ============================================================ tensor-core version
constexpr int kD = 64, kBM = 64, kBN = 64;  // head dim, query rows per CTA, keys per block

__device__ __forceinline__ uint32_t smaddr(const void* p) { return uint32_t(__cvta_generic_to_shared(p)); }
// 64-column bf16 tile, 128-byte rows, 16-byte chunks XOR-swizzled by the row
__device__ __forceinline__ uint32_t swz(int row, int col) {
  return uint32_t(row) * 128u + (uint32_t(((col >> 3) ^ (row & 7))) << 4) + uint32_t(col & 7) * 2u;
}
__device__ __forceinline__ void cp16(uint32_t dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
__device__ __forceinline__ void ldsm4(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}
__device__ __forceinline__ void ldsm4t(uint32_t addr, uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.trans.shared.b16 {%0,%1,%2,%3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3)
               : "r"(addr));
}
__device__ __forceinline__ void mma(float (&c)[4], uint32_t a0, uint32_t a1, uint32_t a2, uint32_t a3, uint32_t b0,
                                    uint32_t b1) {
  asm volatile("mma.sync.aligned.m16n8k16.row.col.f32.bf16.bf16.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
               "{%0,%1,%2,%3};"
               : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
               : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}
__device__ __forceinline__ uint32_t pack_bf16(float lo, float hi) {
  __nv_bfloat162 h = __floats2bfloat162_rn(lo, hi);
  return *reinterpret_cast<uint32_t*>(&h);
}

// load rows [r0, r0+64) x 64 columns (col0 ..) of a [rows, ld] bf16 matrix into a swizzled tile
__device__ __forceinline__ void load_tile(uint8_t* tile, const bf16* base, int64_t ld, int tid) {
#pragma unroll
  for (int it = 0; it < 4; ++it) {
    const int idx = tid + 128 * it;  // 512 16-byte chunks
    const int r = idx >> 3, ch = idx & 7;
    cp16(smaddr(tile) + swz(r, ch * 8), base + int64_t(r) * ld + ch * 8);
  }
}

// A fragments (row-major 16 x 16 at rows m0.., cols k0..) from a [row][col] tile
__device__ __forceinline__ void lda(const uint8_t* tile, int m0, int k0, int lane, uint32_t (&a)[4]) {
  const int r = m0 + (lane & 15), c = k0 + ((lane >> 4) << 3);
  ldsm4(smaddr(tile) + swz(r, c), a[0], a[1], a[2], a[3]);
}
// B fragments for two n-tiles (n0.., n0+8..) x one 16-k step from an [n][k] tile
__device__ __forceinline__ void ldb_nk(const uint8_t* tile, int n0, int k0, int lane, uint32_t (&b)[4]) {
  const int r = n0 + (lane & 7) + ((lane >> 4) << 3), c = k0 + (((lane >> 3) & 1) << 3);
  ldsm4(smaddr(tile) + swz(r, c), b[0], b[1], b[2], b[3]);  // b0,b1 of n0; b0,b1 of n0+8
}
// B fragments for two n-tiles from a [k][n] tile (transposed load)
__device__ __forceinline__ void ldb_kn(const uint8_t* tile, int n0, int k0, int lane, uint32_t (&b)[4]) {
  const int r = k0 + (lane & 7) + (((lane >> 3) & 1) << 3), c = n0 + ((lane >> 4) << 3);
  ldsm4t(smaddr(tile) + swz(r, c), b[0], b[1], b[2], b[3]);
}
// ---------------------------------------------------------------- forward
// grid (seq/64, heads, nb); 4 warps x 16 query rows
__global__ void __launch_bounds__(128) fa_fwd(AttnArgs A) {
  __shared__ __align__(128) uint8_t sQ[kBM * 128];
  __shared__ __align__(128) uint8_t sK[2][kBN * 128];
  __shared__ __align__(128) uint8_t sV[2][kBN * 128];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int qb = blockIdx.x, a = blockIdx.y, b = blockIdx.z;
  const int S = A.seq;
  const int64_t ld = A.ld;
  const uint32_t step = A.step_ptr ? *A.step_ptr : A.step;
  const bf16* Q = static_cast<const bf16*>(A.q) + (int64_t(b) * S + qb * kBM) * ld + a * kD;
  const bf16* K = static_cast<const bf16*>(A.k) + int64_t(b) * S * ld + a * kD;
  const bf16* V = static_cast<const bf16*>(A.v) + int64_t(b) * S * ld + a * kD;
  load_tile(sQ, Q, ld, tid);
  load_tile(sK[0], K, ld, tid);
  load_tile(sV[0], V, ld, tid);
  cp_commit();
  const int nkb = S / kBN;
  const float sl2 = A.alpha * kLog2e;
  float o[8][4] = {};
  float m[2] = {-INFINITY, -INFINITY}, l[2] = {0.f, 0.f};
  uint32_t qa[4][4];
  const int r_lo = warp * 16 + (lane >> 2);  // rows of this thread within the CTA tile
  // element index of (this quad's row r_lo, key 0) in the [b,a,s,s] probabilities
  const uint64_t equad = ((uint64_t(A.b0 + b) * A.heads + a) * S + qb * kBM + r_lo) * uint64_t(S);
  for (int kb = 0; kb < nkb; ++kb) {
    if (kb + 1 < nkb) {
      load_tile(sK[(kb + 1) & 1], K + int64_t(kb + 1) * kBN * ld, ld, tid);
      load_tile(sV[(kb + 1) & 1], V + int64_t(kb + 1) * kBN * ld, ld, tid);
    }
    cp_commit();
    cp_wait<1>();
    __syncthreads();
    if (kb == 0) {
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) lda(sQ, warp * 16, kk * 16, lane, qa[kk]);
    }
    const uint8_t* k_t = sK[kb & 1];
    const uint8_t* v_t = sV[kb & 1];
    float s[8][4] = {};
#pragma unroll
    for (int nn = 0; nn < 4; ++nn)
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        uint32_t bb[4];
        ldb_nk(k_t, nn * 16, kk * 16, lane, bb);
        mma(s[2 * nn], qa[kk][0], qa[kk][1], qa[kk][2], qa[kk][3], bb[0], bb[1]);
        mma(s[2 * nn + 1], qa[kk][0], qa[kk][1], qa[kk][2], qa[kk][3], bb[2], bb[3]);
      }
    // online softmax (base 2), rows r_lo (c0,c1) and r_lo + 8 (c2,c3)
    float mx[2] = {m[0], m[1]};
#pragma unroll
    for (int n = 0; n < 8; ++n) {
      mx[0] = fmaxf(mx[0], fmaxf(s[n][0], s[n][1]) * sl2);
      mx[1] = fmaxf(mx[1], fmaxf(s[n][2], s[n][3]) * sl2);
    }
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      mx[h] = fmaxf(mx[h], __shfl_xor_sync(0xffffffffu, mx[h], 1));
      mx[h] = fmaxf(mx[h], __shfl_xor_sync(0xffffffffu, mx[h], 2));
    }
    const float corr0 = ex2(m[0] - mx[0]), corr1 = ex2(m[1] - mx[1]);
    m[0] = mx[0];
    m[1] = mx[1];
    l[0] *= corr0;
    l[1] *= corr1;
#pragma unroll
    for (int n = 0; n < 8; ++n) {
      o[n][0] *= corr0;
      o[n][1] *= corr0;
      o[n][2] *= corr1;
      o[n][3] *= corr1;
    }
    uint32_t pa[4][4];  // P as A fragments of the PV product (k = keys)
    uint32_t mw[2][2] = {{0u, 0u}, {0u, 0u}};  // [word of the 64-key block][row r_lo / r_lo + 8]
#pragma unroll
    for (int n = 0; n < 8; ++n) {
      float p0 = ex2(s[n][0] * sl2 - m[0]), p1 = ex2(s[n][1] * sl2 - m[0]);
      float p2 = ex2(s[n][2] * sl2 - m[1]), p3 = ex2(s[n][3] * sl2 - m[1]);
      l[0] += p0 + p1;
      l[1] += p2 + p3;
      bool kp[4] = {true, true, true, true};
      if (A.p > 0.f) {
        quad_keep(equad + uint64_t(kb * kBN + n * 8), uint64_t(S), A.seed, step, A.thr, kp);
        p0 = kp[0] ? p0 : 0.f;
        p1 = kp[1] ? p1 : 0.f;
        p2 = kp[2] ? p2 : 0.f;
        p3 = kp[3] ? p3 : 0.f;
      }
      {
        const int bit = (n & 3) * 8 + 2 * (lane & 3);
        mw[n >> 2][0] |= (uint32_t(kp[0]) << bit) | (uint32_t(kp[1]) << (bit + 1));
        mw[n >> 2][1] |= (uint32_t(kp[2]) << bit) | (uint32_t(kp[3]) << (bit + 1));
      }
      const int kk = n >> 1;
      if ((n & 1) == 0) {
        pa[kk][0] = pack_bf16(p0, p1);
        pa[kk][1] = pack_bf16(p2, p3);
      } else {
        pa[kk][2] = pack_bf16(p0, p1);
        pa[kk][3] = pack_bf16(p2, p3);
      }
    }
    if (A.mask) {  // OR the quad's bits; lane 0 of the quad stores this block's 2 words per row
#pragma unroll
      for (int w = 0; w < 2; ++w)
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          mw[w][h] |= __shfl_xor_sync(0xffffffffu, mw[w][h], 1);
          mw[w][h] |= __shfl_xor_sync(0xffffffffu, mw[w][h], 2);
        }
      if ((lane & 3) == 0) {
        uint32_t* m0 = A.mask + ((int64_t(b) * A.heads + a) * S + qb * kBM + r_lo) * (S / 32) + kb * 2;
        m0[0] = mw[0][0];
        m0[1] = mw[1][0];
        m0[8 * (S / 32)] = mw[0][1];
        m0[8 * (S / 32) + 1] = mw[1][1];
      }
    }
#pragma unroll
    for (int nn = 0; nn < 4; ++nn)
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        uint32_t bb[4];
        ldb_kn(v_t, nn * 16, kk * 16, lane, bb);
        mma(o[2 * nn], pa[kk][0], pa[kk][1], pa[kk][2], pa[kk][3], bb[0], bb[1]);
        mma(o[2 * nn + 1], pa[kk][0], pa[kk][1], pa[kk][2], pa[kk][3], bb[2], bb[3]);
      }
    __syncthreads();
  }
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    l[h] += __shfl_xor_sync(0xffffffffu, l[h], 1);
    l[h] += __shfl_xor_sync(0xffffffffu, l[h], 2);
  }
  const float keep_scale = A.p > 0.f ? 1.f / (1.f - A.p) : 1.f;
  const float inv0 = keep_scale / l[0], inv1 = keep_scale / l[1];
  const int q0 = qb * kBM + r_lo;
  if (A.c) {
    bf16* C = static_cast<bf16*>(A.c) + (int64_t(b) * S + q0) * ld + a * kD;
#pragma unroll
    for (int n = 0; n < 8; ++n) {
      const int col = n * 8 + 2 * (lane & 3);
      *reinterpret_cast<uint32_t*>(C + col) = pack_bf16(o[n][0] * inv0, o[n][1] * inv0);
      *reinterpret_cast<uint32_t*>(C + 8 * ld + col) = pack_bf16(o[n][2] * inv1, o[n][3] * inv1);
    }
  }
  if (A.lse && (lane & 3) == 0) {
    float* L = A.lse + (int64_t(b) * A.heads + a) * S + q0;
    L[0] = (m[0] + log2f(l[0])) * kLn2;
    L[8] = (m[1] + log2f(l[1])) * kLn2;
  }
}

// ---------------------------------------------------------------- backward: dQ (+ D)
// grid (seq/64, heads, nb); 4 warps x 16 query rows; loops over key blocks
__global__ void __launch_bounds__(128) fa_bwd_dq(AttnArgs A) {
  __shared__ __align__(128) uint8_t sQ[kBM * 128];
  __shared__ __align__(128) uint8_t sdO[kBM * 128];
  __shared__ __align__(128) uint8_t sK[2][kBN * 128];
  __shared__ __align__(128) uint8_t sV[2][kBN * 128];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int qb = blockIdx.x, a = blockIdx.y, b = blockIdx.z;
  const int S = A.seq;
  const int64_t ld = A.ld;
  const int64_t qrow0 = (int64_t(b) * S + qb * kBM) * ld + a * kD;
  const bf16* Q = static_cast<const bf16*>(A.q) + qrow0;
  const bf16* dO = static_cast<const bf16*>(A.dc) + qrow0;
  const bf16* O = static_cast<const bf16*>(A.c) + qrow0;
  const bf16* K = static_cast<const bf16*>(A.k) + int64_t(b) * S * ld + a * kD;
  const bf16* V = static_cast<const bf16*>(A.v) + int64_t(b) * S * ld + a * kD;
  load_tile(sQ, Q, ld, tid);
  load_tile(sdO, dO, ld, tid);
  load_tile(sK[0], K, ld, tid);
  load_tile(sV[0], V, ld, tid);
  cp_commit();
  const int r_lo = warp * 16 + (lane >> 2);
  const int q0 = qb * kBM + r_lo;
  // D_i = dO_i . O_i (the softmax-backward row term, with dropout folded in)
  float Dr[2];
  {
    const bf16* o0 = O + int64_t(r_lo) * ld;
    const bf16* g0 = dO + int64_t(r_lo) * ld;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      float acc = 0.f;
      for (int c = 2 * (lane & 3); c < kD; c += 8) {
        const float2 x = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(o0 + h * 8 * ld + c));
        const float2 y = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(g0 + h * 8 * ld + c));
        acc += x.x * y.x + x.y * y.y;
      }
      acc += __shfl_xor_sync(0xffffffffu, acc, 1);
      acc += __shfl_xor_sync(0xffffffffu, acc, 2);
      Dr[h] = acc;
    }
  }
  const float* Lrow = A.lse + (int64_t(b) * A.heads + a) * S + q0;
  const float lse2[2] = {Lrow[0] * kLog2e, Lrow[8] * kLog2e};
  const float sl2 = A.alpha * kLog2e;
  const float keep_scale = A.p > 0.f ? 1.f / (1.f - A.p) : 1.f;
  const uint32_t* mrow0 = A.mask + ((int64_t(b) * A.heads + a) * S + q0) * (S / 32);
  const uint32_t* mrow1 = mrow0 + 8 * (S / 32);
  uint32_t qa[4][4], ga[4][4];
  float dq[8][4] = {};
  float rsum[2] = {0.f, 0.f};  // row sums of dS (D consistency, below)
  const int nkb = S / kBN;
  for (int kb = 0; kb < nkb; ++kb) {
    if (kb + 1 < nkb) {
      load_tile(sK[(kb + 1) & 1], K + int64_t(kb + 1) * kBN * ld, ld, tid);
      load_tile(sV[(kb + 1) & 1], V + int64_t(kb + 1) * kBN * ld, ld, tid);
    }
    cp_commit();
    cp_wait<1>();
    __syncthreads();
    if (kb == 0) {
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        lda(sQ, warp * 16, kk * 16, lane, qa[kk]);
        lda(sdO, warp * 16, kk * 16, lane, ga[kk]);
      }
    }
    const uint8_t* k_t = sK[kb & 1];
    const uint8_t* v_t = sV[kb & 1];
    float s[8][4] = {}, dp[8][4] = {};
#pragma unroll
    for (int nn = 0; nn < 4; ++nn)
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        uint32_t bb[4], bv[4];
        ldb_nk(k_t, nn * 16, kk * 16, lane, bb);
        ldb_nk(v_t, nn * 16, kk * 16, lane, bv);
        mma(s[2 * nn], qa[kk][0], qa[kk][1], qa[kk][2], qa[kk][3], bb[0], bb[1]);
        mma(s[2 * nn + 1], qa[kk][0], qa[kk][1], qa[kk][2], qa[kk][3], bb[2], bb[3]);
        mma(dp[2 * nn], ga[kk][0], ga[kk][1], ga[kk][2], ga[kk][3], bv[0], bv[1]);
        mma(dp[2 * nn + 1], ga[kk][0], ga[kk][1], ga[kk][2], ga[kk][3], bv[2], bv[3]);
      }
    uint32_t da[4][4];  // dS as A fragments (k = keys)
#pragma unroll
    for (int n = 0; n < 8; ++n) {
      float v4[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float pr = ex2(s[n][e] * sl2 - lse2[e >> 1]);
        v4[e] = pr;
      }
      float d0 = dp[n][0] * keep_scale, d1 = dp[n][1] * keep_scale, d2 = dp[n][2] * keep_scale,
            d3 = dp[n][3] * keep_scale;
      if (A.p > 0.f) {
        const int key = kb * kBN + n * 8 + 2 * (lane & 3);
        const uint32_t w0 = mrow0[key >> 5] >> (key & 31), w1 = mrow1[key >> 5] >> (key & 31);
        d0 = (w0 & 1u) ? d0 : 0.f;
        d1 = (w0 & 2u) ? d1 : 0.f;
        d2 = (w1 & 1u) ? d2 : 0.f;
        d3 = (w1 & 2u) ? d3 : 0.f;
      }
      const float s0 = v4[0] * (d0 - Dr[0]), s1 = v4[1] * (d1 - Dr[0]);
      const float s2 = v4[2] * (d2 - Dr[1]), s3 = v4[3] * (d3 - Dr[1]);
      rsum[0] += s0 + s1;
      rsum[1] += s2 + s3;
      const int kk = n >> 1;
      if ((n & 1) == 0) {
        da[kk][0] = pack_bf16(s0, s1);
        da[kk][1] = pack_bf16(s2, s3);
      } else {
        da[kk][2] = pack_bf16(s0, s1);
        da[kk][3] = pack_bf16(s2, s3);
      }
    }
#pragma unroll
    for (int nn = 0; nn < 4; ++nn)
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        uint32_t bb[4];
        ldb_kn(k_t, nn * 16, kk * 16, lane, bb);
        mma(dq[2 * nn], da[kk][0], da[kk][1], da[kk][2], da[kk][3], bb[0], bb[1]);
        mma(dq[2 * nn + 1], da[kk][0], da[kk][1], da[kk][2], da[kk][3], bb[2], bb[3]);
      }
    __syncthreads();
  }
  // D for the dK/dV kernel: D_i = sum_j P_ij dP_ij exactly over the P this kernel rebuilt.
  // dO . O differs from it by the bf16 rounding of O, and sum_j dS_ij = sum_j P_ij dP_ij - D_i
  // (sum_j P_ij = 1), so D + sum_j dS_ij is the consistent row term: with it dS has zero row
  // sums and the key-bias gradient keeps its analytic zero (softmax shift invariance).
#pragma unroll
  for (int h = 0; h < 2; ++h) {
    rsum[h] += __shfl_xor_sync(0xffffffffu, rsum[h], 1);
    rsum[h] += __shfl_xor_sync(0xffffffffu, rsum[h], 2);
  }
  if ((lane & 3) == 0) {
    float* Dw = A.ws + (int64_t(b) * A.heads + a) * S + q0;
    Dw[0] = Dr[0] + rsum[0];
    Dw[8] = Dr[1] + rsum[1];
  }
  if (A.dq) {
    bf16* dQ = static_cast<bf16*>(A.dq) + (int64_t(b) * S + q0) * ld + a * kD;
#pragma unroll
    for (int n = 0; n < 8; ++n) {
      const int col = n * 8 + 2 * (lane & 3);
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        uint32_t* pp = reinterpret_cast<uint32_t*>(dQ + h * 8 * ld + col);
        float x = dq[n][2 * h] * A.alpha, y = dq[n][2 * h + 1] * A.alpha;
        if (A.acc_q) {
          const float2 f = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(pp));
          x += f.x;
          y += f.y;
        }
        *pp = pack_bf16(x, y);
      }
    }
  }
}

// ---------------------------------------------------------------- backward: dK, dV
// grid (seq/64 key blocks, heads, nb); warp w owns keys 16w..16w+15; loops over query
// blocks: S = Q K_w^T and dPd = dO V_w^T (queries x 16 keys), P / dS staged in a
// per-warp [query][key] buffer, then dV_w += Pd^T dO and dK_w += dS^T Q.
constexpr int kPS = 48;  // bytes per row of the per-warp [64 q][16 key] staging (ldmatrix conflict-free)

__device__ __forceinline__ void lda_stage_t(const uint8_t* st, int k0, int lane, uint32_t (&a)[4]) {
  // A = X^T (16 keys x 16 queries) from a [query][key] staging buffer, queries k0..k0+15
  const int r = k0 + (lane & 7) + ((lane >> 4) << 3), c = ((lane >> 3) & 1) << 3;
  ldsm4t(smaddr(st) + uint32_t(r * kPS + c * 2), a[0], a[1], a[2], a[3]);
}

constexpr int kDkvSmem = 6 * kBM * 128 + 8 * kBM * kPS;  // K, V, 2 x Q, 2 x dO, 4 x (P, dS) staging

__global__ void __launch_bounds__(128) fa_bwd_dkv(AttnArgs A) {
  extern __shared__ __align__(128) uint8_t dsm[];
  uint8_t* sK = dsm;
  uint8_t* sV = sK + kBN * 128;
  uint8_t* sQ[2] = {sV + kBN * 128, sV + kBN * 128 + kBM * 128};
  uint8_t* sdO[2] = {sQ[1] + kBM * 128, sQ[1] + 2 * kBM * 128};
  uint8_t* sP[4];
  uint8_t* sS[4];
  for (int w = 0; w < 4; ++w) {
    sP[w] = sdO[1] + kBM * 128 + w * kBM * kPS;
    sS[w] = sdO[1] + kBM * 128 + (4 + w) * kBM * kPS;
  }
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int kb = blockIdx.x, a = blockIdx.y, b = blockIdx.z;
  const int S = A.seq;
  const int64_t ld = A.ld;
  const int64_t base = int64_t(b) * S * ld + a * kD;
  const bf16* K = static_cast<const bf16*>(A.k) + base + int64_t(kb) * kBN * ld;
  const bf16* V = static_cast<const bf16*>(A.v) + base + int64_t(kb) * kBN * ld;
  const bf16* Q = static_cast<const bf16*>(A.q) + base;
  const bf16* dO = static_cast<const bf16*>(A.dc) + base;
  const float* L = A.lse + (int64_t(b) * A.heads + a) * S;
  const float* D = A.ws + (int64_t(b) * A.heads + a) * S;
  load_tile(sK, K, ld, tid);
  load_tile(sV, V, ld, tid);
  load_tile(sQ[0], Q, ld, tid);
  load_tile(sdO[0], dO, ld, tid);
  cp_commit();
  const float sl2 = A.alpha * kLog2e;
  const float keep_scale = A.p > 0.f ? 1.f / (1.f - A.p) : 1.f;
  const int key_w = warp * 16;  // this warp's keys within the block
  float dk[8][4] = {}, dv[8][4] = {};
  uint8_t* stP = sP[warp];
  uint8_t* stS = sS[warp];
  const int nqb = S / kBM;
  for (int qb = 0; qb < nqb; ++qb) {
    if (qb + 1 < nqb) {
      load_tile(sQ[(qb + 1) & 1], Q + int64_t(qb + 1) * kBM * ld, ld, tid);
      load_tile(sdO[(qb + 1) & 1], dO + int64_t(qb + 1) * kBM * ld, ld, tid);
    }
    cp_commit();
    cp_wait<1>();
    __syncthreads();
    const uint8_t* q_t = sQ[qb & 1];
    const uint8_t* g_t = sdO[qb & 1];
    // S (64 queries x 16 keys) and dPd, as 4 m-tiles x 2 n-tiles
    float s[4][2][4] = {}, dp[4][2][4] = {};
#pragma unroll
    for (int mt = 0; mt < 4; ++mt)
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        uint32_t qa[4], ga[4], bk[4], bv[4];
        lda(q_t, mt * 16, kk * 16, lane, qa);
        lda(g_t, mt * 16, kk * 16, lane, ga);
        ldb_nk(sK, key_w, kk * 16, lane, bk);
        ldb_nk(sV, key_w, kk * 16, lane, bv);
        mma(s[mt][0], qa[0], qa[1], qa[2], qa[3], bk[0], bk[1]);
        mma(s[mt][1], qa[0], qa[1], qa[2], qa[3], bk[2], bk[3]);
        mma(dp[mt][0], ga[0], ga[1], ga[2], ga[3], bv[0], bv[1]);
        mma(dp[mt][1], ga[0], ga[1], ga[2], ga[3], bv[2], bv[3]);
      }
    // P, Pd, dS -> per-warp staging [query][key]
#pragma unroll
    for (int mt = 0; mt < 4; ++mt) {
      float l2[2], Dq[2];
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int qg = qb * kBM + mt * 16 + (lane >> 2) + 8 * h;
        l2[h] = L[qg] * kLog2e;
        Dq[h] = D[qg];
      }
#pragma unroll
      for (int nt = 0; nt < 2; ++nt) {
        bool kp[4] = {true, true, true, true};
        const int kl = nt * 8 + 2 * (lane & 3);  // key within the warp's 16
        if (A.p > 0.f) {
          const int key = kb * kBN + key_w + kl;
          const uint32_t* m0 = A.mask + ((int64_t(b) * A.heads + a) * S + qb * kBM + mt * 16 + (lane >> 2)) * (S / 32);
          const uint32_t w0 = m0[key >> 5] >> (key & 31), w1 = m0[8 * (S / 32) + (key >> 5)] >> (key & 31);
          kp[0] = w0 & 1u;
          kp[1] = w0 & 2u;
          kp[2] = w1 & 1u;
          kp[3] = w1 & 2u;
        }
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int ql = mt * 16 + (lane >> 2) + 8 * h;  // query within the block
          float p0 = ex2(s[mt][nt][2 * h] * sl2 - l2[h]), p1 = ex2(s[mt][nt][2 * h + 1] * sl2 - l2[h]);
          float d0 = dp[mt][nt][2 * h] * keep_scale, d1 = dp[mt][nt][2 * h + 1] * keep_scale;
          float pd0 = p0 * keep_scale, pd1 = p1 * keep_scale;
          if (!kp[2 * h]) d0 = pd0 = 0.f;
          if (!kp[2 * h + 1]) d1 = pd1 = 0.f;
          *reinterpret_cast<uint32_t*>(stP + ql * kPS + kl * 2) = pack_bf16(pd0, pd1);
          *reinterpret_cast<uint32_t*>(stS + ql * kPS + kl * 2) = pack_bf16(p0 * (d0 - Dq[h]), p1 * (d1 - Dq[h]));
        }
      }
    }
    __syncwarp();
    // dV_w += Pd^T dO, dK_w += dS^T Q (k = the 64 queries)
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
      uint32_t pa[4], sa[4];
      lda_stage_t(stP, kk * 16, lane, pa);
      lda_stage_t(stS, kk * 16, lane, sa);
#pragma unroll
      for (int nn = 0; nn < 4; ++nn) {
        uint32_t bg[4], bq[4];
        ldb_kn(g_t, nn * 16, kk * 16, lane, bg);
        ldb_kn(q_t, nn * 16, kk * 16, lane, bq);
        mma(dv[2 * nn], pa[0], pa[1], pa[2], pa[3], bg[0], bg[1]);
        mma(dv[2 * nn + 1], pa[0], pa[1], pa[2], pa[3], bg[2], bg[3]);
        mma(dk[2 * nn], sa[0], sa[1], sa[2], sa[3], bq[0], bq[1]);
        mma(dk[2 * nn + 1], sa[0], sa[1], sa[2], sa[3], bq[2], bq[3]);
      }
    }
    __syncthreads();
  }
  const int k0 = kb * kBN + key_w + (lane >> 2);
#pragma unroll
  for (int n = 0; n < 8; ++n) {
    const int col = n * 8 + 2 * (lane & 3);
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int64_t off = base + int64_t(k0 + 8 * h) * ld + col;
      if (A.dk) {
        uint32_t* pp = reinterpret_cast<uint32_t*>(static_cast<bf16*>(A.dk) + off);
        float x = dk[n][2 * h] * A.alpha, y = dk[n][2 * h + 1] * A.alpha;
        if (A.acc_k) {
          const float2 f = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(pp));
          x += f.x;
          y += f.y;
        }
        *pp = pack_bf16(x, y);
      }
      if (A.dv) {
        uint32_t* pp = reinterpret_cast<uint32_t*>(static_cast<bf16*>(A.dv) + off);
        float x = dv[n][2 * h], y = dv[n][2 * h + 1];
        if (A.acc_v) {
          const float2 f = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(pp));
          x += f.x;
          y += f.y;
        }
        *pp = pack_bf16(x, y);
      }
    }
  }
}

bool tc_eligible(const AttnArgs& A) {
  return A.dtype == BF16 && A.d == kD && A.seq % 64 == 0 && A.ld % 8 == 0 && A.nb > 0 &&
         reinterpret_cast<uintptr_t>(A.q) % 16 == 0 && reinterpret_cast<uintptr_t>(A.k) % 16 == 0 &&
         reinterpret_cast<uintptr_t>(A.v) % 16 == 0;
}

void fill_thr(AttnArgs& A) { A.thr = dropout_thr16(A.p); }

}  // namespace

bool attention_tc_eligible(const AttnArgs& A) { return tc_eligible(A); }

void attention_simt(const AttnArgs& in, bool bwd, cudaStream_t st) {
  AttnArgs A = in;
  fill_thr(A);
  dim3 grid(A.seq, A.heads, A.nb);
  if (!bwd) {
    if (A.dtype == BF16) attn_fwd_simt<bf16><<<grid, 128, A.seq * sizeof(float), st>>>(A);
    else attn_fwd_simt<float><<<grid, 128, A.seq * sizeof(double), st>>>(A);
  } else if (A.dtype == BF16) {
    attn_bwd_q_simt<bf16><<<grid, 128, 2 * A.seq * sizeof(float), st>>>(A);
    attn_bwd_kv_simt<bf16><<<grid, 128, 2 * A.seq * sizeof(float), st>>>(A);
  } else {
    attn_bwd_q_simt<float><<<grid, 128, 2 * A.seq * sizeof(double), st>>>(A);
    attn_bwd_kv_simt<float><<<grid, 128, 2 * A.seq * sizeof(double), st>>>(A);
  }
}

void attention_fwd(const AttnArgs& in, cudaStream_t st) {
  AttnArgs A = in;
  fill_thr(A);
  dim3 grid(A.seq, A.heads, A.nb);
  if (!A.no_tc5 && attention_fwd_tc5(A, st)) return;  // tcgen05 (attention_tc.cu)
  if (tc_eligible(A)) {
    fa_fwd<<<dim3(A.seq / kBM, A.heads, A.nb), 128, 0, st>>>(A);
  } else if (A.dtype == BF16) {
    attn_fwd_simt<bf16><<<grid, 128, A.seq * sizeof(float), st>>>(A);
  } else {
    attn_fwd_simt<float><<<grid, 128, A.seq * sizeof(double), st>>>(A);
  }
}

void attention_bwd(const AttnArgs& in, cudaStream_t st) {
  AttnArgs A = in;
  fill_thr(A);
  dim3 grid(A.seq, A.heads, A.nb);
  if (!A.no_tc5 && attention_bwd_tc5(A, st)) return;  // tcgen05 (attention_tc.cu)
  if (tc_eligible(A)) {
    fa_bwd_dq<<<dim3(A.seq / kBM, A.heads, A.nb), 128, 0, st>>>(A);
    static bool attr = false;
    if (!attr) {
      cudaFuncSetAttribute(fa_bwd_dkv, cudaFuncAttributeMaxDynamicSharedMemorySize, kDkvSmem);
      attr = true;
    }
    fa_bwd_dkv<<<dim3(A.seq / kBN, A.heads, A.nb), 128, kDkvSmem, st>>>(A);
  } else if (A.dtype == BF16) {
    attn_bwd_q_simt<bf16><<<grid, 128, 2 * A.seq * sizeof(float), st>>>(A);
    attn_bwd_kv_simt<bf16><<<grid, 128, 2 * A.seq * sizeof(float), st>>>(A);
  } else {
    attn_bwd_q_simt<float><<<grid, 128, 2 * A.seq * sizeof(double), st>>>(A);
    attn_bwd_kv_simt<float><<<grid, 128, 2 * A.seq * sizeof(double), st>>>(A);
  }
}

}  // namespace tsk
