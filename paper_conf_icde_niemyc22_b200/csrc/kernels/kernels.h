// Host-side launchers of the sm_100a kernel library (all asynchronous on `st`).
// Every micro-op of the augmented schedule maps to one or more of these; the
// pointers are micro-tensor views (a split shares storage, only the
// pointer changes).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <vector>

namespace tsk {

enum DType : int { F32 = 0, BF16 = 1 };

// Logical A[M,K], B[N,K]; element (m,k) of A at a + (mn ? k*lda + m : m*lda + k)
// + b1*bs1 + b2*bs2 (elements).  C[m,n] = alpha*sum_k A B + bias[n] + beta*C.
struct GemmOperand {
  const void* ptr = nullptr;
  int64_t ld = 0;
  bool mn_major = false;
  int64_t bs1 = 0, bs2 = 0;
};
constexpr int kMaxGroups = 3;
struct GemmArgs {
  int M = 0, N = 0, K = 0, nb1 = 1, nb2 = 1;
  int in_dtype = BF16;
  GemmOperand a, b;
  void* c = nullptr;
  int64_t ldc = 0, cbs1 = 0, cbs2 = 0;
  int c_dtype = BF16;
  float alpha = 1.f, beta = 0.f;
  const void* bias = nullptr;
  int bias_dtype = BF16;
  // fused epilogue (bf16 C, beta = 0): 1 = GELU forward, C = U = alpha AB + bias and
  // aux = gelu(U) (the linear -> gelu pair of one micro-op); 2 = GELU backward, C = dU =
  // bf16(alpha AB) * gelu'(aux) with aux = U (the dX product of the layer after a gelu).
  // Values pass through bf16 exactly where the separate kernels would store them.
  // 3 = residual add, C = U = alpha AB + bias and aux2 = bf16(U) + aux (the linear -> add
  // pair whose add reads the linear's output and a residual aux, e.g. res1 = proj + x).
  int epi = 0;
  void* aux = nullptr;
  int64_t ldaux = 0;
  void* aux2 = nullptr;  // epi 3 output (row-major, leading dimension ldaux2)
  int64_t ldaux2 = 0;
  // grouped product (tcgen05 path only, unbatched, epi 0, beta 0 or 1): `groups` equal
  // slices along gdim, M/N/K being the totals.  gdim 1 (N): C_g = A B_g^T + bias_g, per
  // group bg/cg/biasg, shared a; gdim 2 (K): C = sum_g A_g B_g^T, per group ag/bg, shared
  // c; gdim 3 (M): C_g = A_g B^T, per group ag/cg, shared b.  Used to run the q/k/v
  // linears of one micro-op (same input X) as one launch.
  int groups = 1, gdim = 0;
  GemmOperand ag[kMaxGroups], bg[kMaxGroups];
  void* cg[kMaxGroups] = {nullptr, nullptr, nullptr};
  const void* biasg[kMaxGroups] = {nullptr, nullptr, nullptr};
};

// Returns false (and leaves nothing launched) when the shape/alignment does not
// fit the tcgen05/TMA path; gemm() then uses the SIMT kernel.
bool gemm_tc(const GemmArgs& g, cudaStream_t st);
void gemm_simt(const GemmArgs& g, cudaStream_t st);
void gemm(const GemmArgs& g, cudaStream_t st);
int64_t gemm_tc_launches();
// tile configuration of the last gemm_tc launch (tests / tools): width bn of a tile,
// cg = CTAs per tile (2: cta_group::2 pair, 256 rows), split-K factor, work units, SMs,
// co-resident CTA pairs, first half-width tail unit (= units when none)
struct GemmConfig {
  int bn, cg, ksplit, units, sms, pair_slots, split_from;
};
GemmConfig gemm_tc_last_config();
// 0: cost-model choice; 1: single-CTA tiles only; 2: CTA pairs whenever M > 128, N > 64;
// + 4: no half-width tail units
void gemm_tc_set_mode(int mode);
// Per-launch timing of GEMMs (eager profiling only): while enabled, gemm() brackets
// every launch with CUDA events on its stream and records the algorithmic FLOP.
struct GemmRecord {
  cudaEvent_t start, stop;
  double flop;
  int M, N, K, batch, tc;
  int kind;   // 0 GEMM, 1 conv fprop, 2 conv dgrad, 3 conv wgrad
  int flags;  // GEMM: bit0 A MN-major, bit1 B MN-major, bit2 fp32 C, bit3 beta != 0
};
void gemm_records_enable(std::vector<GemmRecord>* sink);
std::vector<GemmRecord>* gemm_records_sink();

// ---- convolution (NHWC activations, KRSC weights; one micro-op = n samples) ------
// Implicit GEMM (conv_tc.cu): fprop M = n*P*Q, N = K, Kg = R*S*C; dgrad M = n*H*W,
// N = C, Kg = R*S*K; wgrad M = R*S*C, N = K, Kg = n*P*Q (split-K, fp32 out).
struct ConvArgs {
  int dtype = BF16;
  int n = 0, H = 0, W = 0, C = 0, K = 0, R = 0, S = 0, P = 0, Q = 0, stride = 1, pad = 0;
  const void* x = nullptr;   // [n,H,W,C]
  const void* w = nullptr;   // [K,R,S,C]
  const void* dy = nullptr;  // [n,P,Q,K]
};
// y[n,P,Q,K] = conv(x, w) (+ bias[K]) — bias in the graph dtype
void conv_fprop(const ConvArgs& a, void* y, const void* bias, cudaStream_t st);
// dx[n,H,W,C] (+)= conv_transpose(dy, w)
void conv_dgrad(const ConvArgs& a, void* dx, int acc, cudaStream_t st);
// dw[K,R,S,C] (fp32) (+)= sum over the micro-op's pixels of dy (x) im2col(x)
void conv_wgrad(const ConvArgs& a, float* dw, int acc, cudaStream_t st);
// tcgen05 path; false when the shape/alignment is not eligible (then SIMT)
bool conv_tc(int mode, const ConvArgs& a, void* out, const void* bias, int acc, cudaStream_t st);
// TMA-fed variant for C % 64 == 0, K % 64 == 0, stride <= 2 (tried first by conv_tc)
bool conv_tma(int mode, const ConvArgs& a, void* out, const void* bias, int acc, cudaStream_t st);
// the cp.async gather kernel alone (tests; conv_tc tries conv_tma first)
bool conv_gather(int mode, const ConvArgs& a, void* out, const void* bias, int acc, cudaStream_t st);
void conv_simt(int mode, const ConvArgs& a, void* out, const void* bias, int acc, cudaStream_t st);

// ---- batch normalisation over all pieces of a split tensor ----------
// A piece list: `np` pointers, each holding `rows[i]` rows of C channels.
struct PieceList {
  static constexpr int kMax = 16;
  const void* ptr[kMax];
  int64_t rows[kMax];
  int np = 0;
};
bool bn_supported(int dt, int C);  // whole 16-byte channel vectors, <= 256 vectors per row
// stats[0:C] = mean, stats[C:2C] = rstd over every row of every piece (fp64 final reduce)
void bn_stats(int dt, const PieceList& x, int C, float eps, float* ws, uint64_t ws_bytes, float* stats,
              cudaStream_t st);
// y = (x - mean) * rstd * gamma + beta on one micro-op's rows
void bn_apply(int dt, const void* x, const float* stats, const void* gamma, const void* beta, void* y, int64_t rows,
              int C, cudaStream_t st);
// full-batch sums: stats[2C:3C] = sum dy*gamma, stats[3C:4C] = sum dy*gamma*xhat;
// dgamma (+)= sum dy*xhat, dbeta (+)= sum dy
void bn_bwd_sums(int dt, const PieceList& dy, const PieceList& x, const void* gamma, int C, float* ws,
                 uint64_t ws_bytes, float* stats, float* dgamma, float* dbeta, int pacc, cudaStream_t st);
// dx (+)= rstd * (dy*gamma - s1/m - xhat*s2/m), m = rows of the whole batch
void bn_bwd_apply(int dt, const void* dy, const void* x, const float* stats, const void* gamma, void* dx, int acc,
                  int64_t rows, int C, int64_t m_total, cudaStream_t st);
// ---- fused attention (attention.cu) -----------------------------
// Q, K, V, C, dC, dQ, dK, dV: [nb*seq, ld] with head a at columns a*d..(a+1)*d;
// lse [nb, heads, seq] fp32; ws >= nb*heads*seq floats (backward row terms D_i).
// Dropout: Philox on the [b,a,s,s] element index with b = b0 + local sample.
struct AttnArgs {
  int dtype = BF16;
  int nb = 0, heads = 0, seq = 0, d = 0;
  int64_t ld = 0;
  const void *q = nullptr, *k = nullptr, *v = nullptr;
  void* c = nullptr;       // forward output (may be null: a replay regenerating only lse)
  float* lse = nullptr;    // forward output (may be null) / backward input
  uint32_t* mask = nullptr;  // dropout keep bits [nb, heads, seq, seq/32]: forward output (may be null) / backward input
  const void* dc = nullptr;
  void *dq = nullptr, *dk = nullptr, *dv = nullptr;
  int acc_q = 0, acc_k = 0, acc_v = 0;
  float alpha = 1.f, p = 0.f;
  uint32_t seed = 0, step = 0, thr = 0;
  // device copy of the step counter: when set, kernels read the dropout step from it at run
  // time (a captured CUDA graph replays with the live value); null = use `step`
  const uint32_t* step_ptr = nullptr;
  int64_t b0 = 0;
  float* ws = nullptr;
  int no_tc5 = 0;  // tests: skip the tcgen05 kernels (mma.sync path instead)
};
bool attention_tc_eligible(const AttnArgs& a);  // bf16, d = 64, seq % 64 == 0 (mma.sync path)
void attention_fwd(const AttnArgs& a, cudaStream_t st);
void attention_bwd(const AttnArgs& a, cudaStream_t st);  // needs a.c (= O), a.lse, a.dc
void attention_simt(const AttnArgs& a, bool bwd, cudaStream_t st);  // CUDA-core kernels only (tests)
// tcgen05 forward (attention_tc.cu): bf16, d = 64, seq % 128 == 0; writes each of C, lse and
// the keep bits whose pointer is set (a replay regenerates only its target); false = not
// eligible (nothing launched).  a.thr must be set.
bool attention_fwd_tc5(const AttnArgs& a, cudaStream_t st);
// tcgen05 backward (same eligibility; needs c, lse, mask, dc, ws)
bool attention_bwd_tc5(const AttnArgs& a, cudaStream_t st);

// ---- pooling (NHWC) ----------------------------------------------------------------
void maxpool_fwd(int dt, const void* x, void* y, int n, int H, int W, int C, int P, int Q, int k, int stride,
                 int pad, cudaStream_t st);
// gradient to the first maximum of each window in row-major order
void maxpool_bwd(int dt, const void* dy, const void* x, void* dx, int acc, int n, int H, int W, int C, int P, int Q,
                 int k, int stride, int pad, cudaStream_t st);
// D-ATTR staging (attr.cu): a band-split NHWC tensor [B, H, W, C] is pieces of hb rows
// (axis 1: piece j = rows [j hb, (j+1) hb) of every sample, [B, hb, W, C]) or of hb columns
// (axis 2: [B, H, hb, C]); an unsplit one is one piece with axis 1, hb = H.
struct BandPieces {
  const void* ptr[16] = {};
  int hb = 0, axis = 1;  // axis 3: channel blocks of hb channels [B, H, W, hb] (D-CH staged merge)
};
// The staged rectangle: rows [rlo, rlo + hs) x columns [clo, clo + ws) of samples [b0, b0 + nb).
struct Rect {
  int b0, nb, rlo, hs, clo, ws;
};
// out[b, r, c', ch] = X[b0 + b, rlo + r, clo + c', ch], fill (0 or -inf) outside X; out [nb, hs, ws, C]
void band_gather(int dt, const BandPieces& x, int H, int W, int C, const Rect& r, int neg_inf_fill, void* out,
                 cudaStream_t st);
// dX[b0 + b, h, w, ch] += src[b, h - rlo, w - clo, ch] for the (h, w) of the rectangle inside X
void band_scatter_add(int dt, const void* src, const BandPieces& dx, int H, int W, int C, const Rect& r,
                      cudaStream_t st);
void avgpool_fwd(int dt, const void* x, void* y, int n, int HW, int C, cudaStream_t st);
void avgpool_bwd(int dt, const void* dy, void* dx, int acc, int n, int HW, int C, cudaStream_t st);

// ---- elementwise (n elements, dtype F32/BF16 for activations) ----------------
void relu_fwd(int dt, const void* x, void* y, int64_t n, cudaStream_t st);
void relu_bwd(int dt, const void* dy, const void* y, void* dx, int acc, int64_t n, cudaStream_t st);
void gelu_fwd(int dt, const void* x, void* y, int64_t n, cudaStream_t st);
void gelu_bwd(int dt, const void* dy, const void* x, void* dx, int acc, int64_t n, cudaStream_t st);
void tanh_fwd(int dt, const void* x, void* y, int64_t n, cudaStream_t st);
void tanh_bwd(int dt, const void* dy, const void* y, void* dx, int acc, int64_t n, cudaStream_t st);
void add_fwd(int dt, const void* a, const void* b, void* y, int64_t n, cudaStream_t st);
// dx (+)= scale * dy (acc: accumulate into dx)
void axpy(int dt, const void* dy, void* dx, int acc, int64_t n, cudaStream_t st);
// add backward: d1 (+)= dy and d2 (+)= dy in one pass (acc flags per output)
void axpy2(int dt, const void* dy, void* d1, int acc1, void* d2, int acc2, int64_t n, cudaStream_t st);
// step_ptr: device step counter read at run time (null: `step`)
void dropout(int dt, const void* x, void* y, int acc, int64_t n, int64_t elem0, float p, uint32_t seed,
             uint32_t step, const uint32_t* step_ptr, cudaStream_t st);
// *counter += 1 on the stream (the session's dropout step, advanced at the end of every step)
void step_advance(uint32_t* counter, cudaStream_t st);
// ---- row ops -----------------------------------------------------------------
void layernorm_fwd(int dt, const void* x, const void* g, const void* b, void* y, int64_t rows, int H,
                   float eps, cudaStream_t st);
// dx (+)= ...; partial dgamma/dbeta rows go to ws, then column_reduce adds them.
void layernorm_bwd(int dt, const void* dy, const void* x, const void* g, void* dx, int acc, float* ws,
                   uint64_t ws_bytes, float* dgamma, float* dbeta, int pacc, int64_t rows, int H, float eps,
                   cudaStream_t st);
// causal: rows are queries i = row % L of [.., L, L] scores; keys j > i get probability 0
void softmax_fwd(int dt, const void* x, void* y, int64_t rows, int L, int causal, cudaStream_t st);
void softmax_bwd(int dt, const void* dy, const void* y, void* dx, int acc, int64_t rows, int L,
                 cudaStream_t st);
// out[n] (+)= sum_r x[r, n] (rows filtered by `filter[r] == fval` when filter != null)
// (deterministic; the last 4 KB of the workspace hold the per-launch completion tickets)
void column_sum(int dt, const void* x, int64_t rows, int N, float* ws, uint64_t ws_bytes, float* out, int acc,
                const int* filter, int fval, cudaStream_t st);
void embed_fwd(int dt, const int* ids, const int* tt, const void* word, const void* pos, const void* type,
               void* y, int64_t rows, int H, int seq, int64_t row0, cudaStream_t st);
void embed_bwd_word(int dt, const void* dy, const int* ids, float* dword, int64_t rows, int H, cudaStream_t st);
// dpos[s, :] (+)= sum over samples of dy rows at position s (rows = nsamp*seq)
void embed_bwd_pos(int dt, const void* dy, float* dpos, int64_t nsamp, int seq, int H, int acc, cudaStream_t st);
void cls_fwd(int dt, const void* x, void* y, int64_t nsamp, int seq, int H, cudaStream_t st);
void cls_bwd(int dt, const void* dy, void* dx, int acc, int64_t nsamp, int seq, int H, cudaStream_t st);
// loss[0] (+)= sum_rows CE / b_global ; dz = (softmax - onehot)/b_global
// (ws: >= rows floats; with many rows (token-level losses) per-row values go there and one
// block sums them in a fixed order)
void xent_fwd(int dt, const void* z, const int* labels, float* loss, int acc, int64_t rows, int C,
              float inv_b, float* ws, cudaStream_t st);
void xent_bwd(int dt, const void* z, const int* labels, void* dz, int acc, int64_t rows, int C, float inv_b,
              cudaStream_t st);
// ---- optimiser / static region ------------------------------------------------
void sgd_update(float* master, const float* grad, int64_t n, float lr, float gscale, cudaStream_t st);
// multi-tensor SGD + bf16 copy refresh: chunk table in device memory (offsets into the slab;
// c_off = ~0 for no copy); chunk starts are 16-byte aligned
struct SgdChunk {
  uint64_t m_off, g_off, c_off;
  int64_t n;
};
void sgd_fused(const SgdChunk* chunks, int n_chunks, char* slab, float lr, float gscale, cudaStream_t st);
void cast_f32_bf16(const float* src, void* dst, int64_t n, cudaStream_t st);
void cast_bf16_f32(const void* src, float* dst, int64_t n, cudaStream_t st);
void scale_f32(float* x, int64_t n, float s, cudaStream_t st);

}  // namespace tsk
