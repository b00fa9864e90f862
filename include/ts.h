/*
 * ts.h — C ABI of the B200-native TSPLIT hot path.
 *
 * TSPLIT (Nie et al., ICDE'22, /root/reference/PAPER.md, cited "P:L<line>")
 * takes a dataflow graph and an available GPU memory M and finds, for every
 * tensor, a configuration {opt, p_num, dim} (§IV-A Eq. 1, §V-A,
 * Fig. 9 `struct config`) so that the memory requirement M_i of every
 * operation stays under M while the added time is small; it then executes the
 * augmented graph (Fig. 10) with a compute stream, a D2H stream and
 * an H2D stream ordered by CUDA events over a pre-allocated pool.
 *
 * Conventions for every entry point:
 *  - Returns ts_status; on failure the out-parameters are untouched and
 *    ts_last_error() returns a thread-local message.
 *  - Arrays passed in are copied at call time (the caller keeps ownership).
 *  - Handles are owned by the caller until the matching *_destroy.
 *  - "device pointer" arguments are CUDA device addresses on the session's
 *    device; "host pointer" arguments are ordinary (pageable or pinned) host
 *    memory.  No torch types cross this boundary.
 *  - Sizes are in bytes unless stated; shapes are row-major (last dim
 *    contiguous).  Tensor ids are indices into the descriptor array.
 */
#ifndef TSPLIT_TS_H
#define TSPLIT_TS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  TS_OK = 0,
  TS_ERR_ARG = 1,         /* bad argument (null pointer, out-of-range id, bad size) */
  TS_ERR_GRAPH = 2,       /* graph does not validate (shape mismatch, cycle, ...)   */
  TS_ERR_INFEASIBLE = 3,  /* Alg. 2 ran out of candidates ("fail because of
                             no more available tensors"); message names the op     */
  TS_ERR_BUDGET = 4,      /* runtime pool overflow: the slab is smaller than the plan */
  TS_ERR_HOST_MEM = 5,    /* pinned host pool allocation failed                     */
  TS_ERR_CUDA = 6,        /* a CUDA runtime/driver call failed (message has it)     */
  TS_ERR_NCCL = 7,        /* NCCL failure                                           */
  TS_ERR_STATE = 8,       /* call made in the wrong order / unsupported here        */
  TS_ERR_NO_GPU = 9       /* no CUDA device: compute entry points refuse (no CPU fallback) */
} ts_status;

typedef enum { TS_F32 = 0, TS_BF16 = 1, TS_I32 = 2 } ts_dtype;
typedef enum { TS_PARAM = 0, TS_INPUT = 1, TS_LABEL = 2, TS_ACT = 3 } ts_kind;
/* Fig. 9 `opt`: memory option of every micro-tensor of a tensor. */
typedef enum { TS_RESIDE = 0, TS_SWAP = 1, TS_RECOMPUTE = 2 } ts_opt;

/* Operation kinds; semantics and attribute layout in DESIGN.md §3. */
typedef enum {
  TS_OP_LINEAR = 0,    /* in X[R,K], W[N,K], b[N]      out Y = X W^T + b              */
  TS_OP_RELU = 1,
  TS_OP_GELU = 2,      /* erf GELU                                                     */
  TS_OP_TANH = 3,
  TS_OP_LAYERNORM = 4, /* in X[R,H], gamma, beta; fattr[0] = eps                       */
  TS_OP_ADD = 5,
  TS_OP_DROPOUT = 6,   /* fattr[0] = p; iattr[0] = seed (Philox4x32-10 key)             */
  TS_OP_SOFTMAX = 7,   /* over the last dim; iattr[0] = 1: causal over [.., s, s] scores
                          (keys j > query i dropped: decoder self-attention, f4)          */
  TS_OP_ATTN_QK = 8,   /* in Q[T,h], K[T,h] out S[b,a,s,s]; iattr {heads, seq}; fattr[0] = alpha */
  TS_OP_ATTN_PV = 9,   /* in P[b,a,s,s], V[T,h] out C[T,h]; iattr {heads, seq}         */
  TS_OP_EMBED = 10,    /* in ids, type_ids (i32 [T]), Wword, Wpos, Wtype; iattr[0] = seq */
  TS_OP_CLS = 11,      /* in X[T,h] out [b,h] (row b*seq); iattr[0] = seq              */
  TS_OP_XENT = 12,     /* in logits[b,C], labels i32[b] out loss f32[1], mean over the
                          global batch                                     */
  TS_OP_CONV2D = 13,   /* in X[N,H,W,C] (NHWC), W[K,R,S,C] (KRSC), [b[K]] out Y[N,P,Q,K];
                          iattr {stride, pad}                                           */
  TS_OP_BATCHNORM = 14,/* in X[...,C], gamma[C], beta[C]; fattr[0] = eps; train-mode
                          batch statistics over all samples even when split (R13)      */
  TS_OP_MAXPOOL = 15,  /* in X[N,H,W,C] out [N,P,Q,C]; iattr {k, stride, pad}           */
  TS_OP_AVGPOOL = 16,  /* global average: in X[N,H,W,C] out [N,C]                       */
  TS_OP_FLATTEN = 17,  /* in X[N,...] out [N, prod(...)] (copy)                          */
  TS_OP_ATTENTION = 18 /* fused attention: in Q[T,h], K[T,h], V[T,h];
                          out C[T,h] = dropout(softmax(alpha Q_h K_h^T)) V_h (heads merged),
                          lse[b,a,s] (f32) and the dropout keep bits [b,a,s,s/32] (i32, key j
                          at bit j%32) — both auxiliary: read only by its own backward, never
                          differentiated; iattr {heads, seq (% 32 == 0), dropout seed},
                          fattr {alpha, p}; keep = Philox on the [b,a,s,s] index (D-RNG)    */
} ts_op_kind;

typedef struct {
  int32_t dtype;       /* ts_dtype */
  int32_t kind;        /* ts_kind  */
  int32_t ndim;        /* 1..6     */
  int64_t shape[6];    /* leading dim of every non-param tensor except the loss is a
                          multiple of `samples` (the split "sample" dim)      */
} ts_tensor_desc;

typedef struct {
  int32_t kind;        /* ts_op_kind */
  int32_t n_in, n_out;
  const int32_t* in;   /* tensor ids */
  const int32_t* out;
  int32_t n_iattr;
  const int64_t* iattr;
  int32_t n_fattr;
  const double* fattr;
} ts_op_desc;

/* Per-tensor configuration: Fig. 9 `struct config` {opt, p_num, dim} plus the
 * prefetch lead of a swapped tensor (swap-in starts `prefetch_lead` compute
 * items before its first backward use; 1 = "the previous computation
 * operation").  dim 0 = the sample dim ("sample dim"); dim 1 = the
 * channel / parameter dim of a 2-D activation [rows, C] (Fig. 6): p_num
 * contiguous column blocks [rows, C/p_num], legal per DESIGN.md reading D-CH (produced by
 * a linear or relu/gelu/tanh, read by a linear as X or relu/gelu/tanh); dim 2 / 3 = the
 * height / width (attribute dims) of a 4-D NHWC activation [B, H, W, C]: p_num
 * bands [B, H/p_num, W, C] (rows [j H/p, (j+1) H/p) of every sample) / [B, H, W/p_num, C],
 * legal per reading D-ATTR
 * (produced by conv2d / maxpool / relu / add / batchnorm, read by those; a window op reads
 * its halo rows through a staged copy — a pool temporary in the trace). */
typedef struct {
  int32_t tensor_id;
  int32_t opt;           /* ts_opt */
  int32_t p_num;         /* 1, 2, 4, 8, 16; must divide `samples` (dim 0), C (dim 1), H (dim 2) or W (dim 3) */
  int32_t dim;
  int32_t prefetch_lead; /* >= 1 */
  int32_t release_lag;   /* swap only (reading D-LAG): the range a swap-out frees
                            returns to the pool after this many compute items behind it
                            (0: at the swap-out), so a later allocation does not wait on
                            the copy (R12); capped before the swap-in */
} ts_tensor_cfg;

typedef struct {
  uint64_t static_bytes;   /* params (fp32 master [+bf16 copy] + fp32 grad) + workspace */
  uint64_t peak_live;      /* static + max_i sum of live micro-tensor bytes (M_i) */
  uint64_t peak_extent;    /* highest pool offset used (includes fragmentation)          */
  uint64_t d2h_bytes;      /* swap-out bytes per step                                    */
  uint64_t h2d_bytes;      /* swap-in bytes per step                                     */
  int64_t n_items;         /* augmented schedule length                                  */
  int64_t n_compute;       /* forward + backward micro-ops                               */
  int64_t n_replay;        /* recompute replays (memory-centric)                 */
  double predicted_s;      /* planner's predicted step time                              */
  double compute_flop;     /* algorithmic FLOP per step incl. replays                    */
  int64_t n_split_tensors; /* tensors with p_num > 1                                     */
  int64_t n_swap_tensors;
  int64_t n_recompute_tensors;
  uint64_t recompute_cache_bytes; /* D-LRU recompute cache limit (0 = memory-centric, Fig. 11) */
} ts_plan_stats_t;

typedef struct {
  int64_t seq;
  int32_t item;          /* augmented-schedule index, -1 = step start           */
  int32_t kind;          /* 0 = ALLOC, 1 = FREE                                 */
  int32_t key;           /* tensor id, or n_tensors + id for its gradient       */
  int32_t piece;         /* micro-tensor index                                   */
  uint64_t offset;       /* byte offset in the pool slab                        */
  uint64_t bytes;        /* unaligned size                                      */
} ts_alloc_event;

/* Hardware model used by the planner (bytes/s and FLOP/s). */
typedef struct {
  double tensor_flops;   /* dense bf16 tensor FLOP/s (MEASURED_PEAKS bf16_tflops_sustained) */
  double simt_flops;     /* fp32 FFMA FLOP/s                                          */
  double hbm_bw;         /* HBM bytes/s (MEASURED_PEAKS hbm_gbs)                       */
  double d2h_bw, h2d_bw; /* PCIe bytes/s, measured per pod                             */
  double launch_s;       /* per-kernel overhead inside a CUDA graph                     */
} ts_hw;

typedef struct ts_graph_s ts_graph_t;
typedef struct ts_profile_s ts_profile_t;
typedef struct ts_plan_s ts_plan_t;
typedef struct ts_session_s ts_session_t;

const char* ts_last_error(void);
const char* ts_version(void);

/* ---- graph (host only) ------------------------------------------------------ */
/* Validates the DFG and builds the Alg. 1 forward schedule (read as
 * ref_cnt -= 1 / == 0); backward = reverse order (R2). */
ts_status ts_graph_define(const ts_tensor_desc* tensors, int32_t n_tensors,
                          const ts_op_desc* ops, int32_t n_ops,
                          int32_t samples, int32_t compute_dtype, ts_graph_t** out);
void ts_graph_destroy(ts_graph_t* g);
/* Writes the forward schedule O (op ids) into order[cap]; *n = number of ops. */
ts_status ts_graph_schedule(const ts_graph_t* g, int32_t* order, int32_t cap, int32_t* n);
ts_status ts_graph_static_bytes(const ts_graph_t* g, uint64_t* out);

/* ---- profile --------------------------------- */
/* Analytic profile from a hardware model: per-op T(p) = launch + max(flop/peak,
 * bytes/bw) for every p in {1,2,4,8,16}. */
ts_status ts_profile_analytic(const ts_graph_t* g, const ts_hw* hw, ts_profile_t** out);
/* Overwrite one measured entry: op id, p_num, forward and backward seconds of the
 * WHOLE op (sum over its p_num micro-ops), e.g. from cudaEvent timing. */
ts_status ts_profile_set(ts_profile_t* pr, int32_t op, int32_t p_num, double fwd_s, double bwd_s);
ts_status ts_profile_set_pcie(ts_profile_t* pr, double d2h_bw, double h2d_bw);
void ts_profile_destroy(ts_profile_t* pr);
/* Measured profile (needs the GPU): for p = 1, 2, 4, ... <= max_p, runs one warm-up and
 * one cudaEvent-timed eager step of the all-reside plan with every activation split p
 * ways, on the caller's scratch `slab` (device, >= the unsplit peak; parameters are
 * zero — op times do not depend on the data), and records each op's forward
 * and backward time (per-item median of three timed steps).  A p the batch does not divide
 * (the sample dim exhausted, Fig. 6) is timed with height bands instead (reading D-ATTR:
 * every group of 4-D activations that can take p bands legally; the ops it splits get that
 * width's times, staging copies included).  p values above max_p, or that no split reaches,
 * extrapolate from the widest measured one (+5 % per doubling: the launch / tail overhead
 * of one more level of micro-ops).  Also measures pinned
 * D2H/H2D bandwidth (256 MiB copies).  `inputs` as in ts_step. */
ts_status ts_profile_measure(const ts_graph_t* g, void* slab, uint64_t slab_bytes, const void* const* inputs,
                             int32_t inputs_on_host, int32_t max_p, ts_profile_t** out);
ts_status ts_profile_get(const ts_profile_t* pr, int32_t op, int32_t p_num, double* fwd_s, double* bwd_s);
ts_status ts_profile_pcie(const ts_profile_t* pr, double* d2h_bw, double* h2d_bw);

/* ---- plan ------------------------------------------------------------------- */
/* All tensors reside, p_num = 1 (the "Base" of P:L304). */
ts_status ts_plan_default(const ts_graph_t* g, ts_plan_t** out);
/* Profiling-based greedy planning (Alg. 2, reconstructed from P:L178/L270, SURVEY
 * R8) under `budget_bytes` for the whole pool (static + dynamic, R4).  `profile`
 * may be NULL (analytic model with B200 defaults).  Returns TS_ERR_INFEASIBLE
 * when no candidate remains. */
ts_status ts_plan(const ts_graph_t* g, uint64_t budget_bytes, const ts_profile_t* profile, ts_plan_t** out);
/* ts_plan with planner options (the breakdown of P:L457-467):
 *   TS_PLAN_NO_SPLIT        "TSPLIT w/o Split": Alg. 2 without split candidates (steps 1, 3 only)
 *   TS_PLAN_MEMORY_CENTRIC  no LRU recompute cache (every backward group regenerates, Fig. 11) */
#define TS_PLAN_NO_SPLIT 1u
#define TS_PLAN_MEMORY_CENTRIC 2u
ts_status ts_plan_ex(const ts_graph_t* g, uint64_t budget_bytes, const ts_profile_t* profile, uint32_t flags,
                     ts_plan_t** out);
ts_status ts_plan_get(const ts_plan_t* p, int32_t tensor_id, ts_tensor_cfg* out);
/* Forced configuration (Fig. 9 set_config); the plan is re-expanded and
 * re-simulated.  Only TS_ACT tensors accept opt != RESIDE or p_num > 1.  p_num divides
 * the samples (dim 0), the columns (dim 1), the height (dim 2) or the width (dim 3).  TS_ERR_ARG (plan
 * unchanged) when a field is out of range or the resulting plan breaks the channel-split
 * (D-CH) or band-split (D-ATTR) rules. */
ts_status ts_plan_set(ts_plan_t* p, const ts_tensor_cfg* cfg);
/* Several configurations applied together, then validated as one (a channel-split chain,
 * e.g. linear -> gelu, is only legal as a whole).  cfgs: host array of n entries, copied.
 * TS_ERR_ARG leaves the plan unchanged. */
ts_status ts_plan_set_many(ts_plan_t* p, const ts_tensor_cfg* cfgs, int32_t n);
ts_status ts_plan_stats(const ts_plan_t* p, ts_plan_stats_t* out);
/* LRU-based recomputation ("execute as the speed-centric manner and abandon the
 * least recently used intermediate tensor once the available memory is not enough";
 * DESIGN.md reading D-LRU).  `cache_bytes` caps the regenerated micro-tensors kept
 * resident across backward groups (checked at the end of each group, least recently used
 * abandoned first); 0 = memory-centric (every backward group regenerates what it reads).
 * ts_plan chooses it (fastest feasible of a small candidate set); this forces one.  The
 * plan is re-expanded and re-simulated; the caller checks the new peak against its budget. */
ts_status ts_plan_set_recompute_cache(ts_plan_t* p, uint64_t cache_bytes);
/* Simulated allocation trace (R3, R11); *n = total events (buf may be NULL). */
ts_status ts_plan_trace(const ts_plan_t* p, ts_alloc_event* buf, uint64_t cap, uint64_t* n);
/* Augmented schedule as int32 quadruples (kind, op, k, aux) — kind 0 F, 1 B, 2 R,
 * 3 SO, 4 SI; aux = piece key for SO/SI (key*65536+piece), else group id. */
ts_status ts_plan_items(const ts_plan_t* p, int32_t* buf, uint64_t cap, uint64_t* n);
/* Data-parallel gradient buckets of this plan: parameters grouped, in
 * the order their gradients become final in the augmented schedule, into buckets of at
 * least bucket_bytes (the session uses 32 MiB).  buf receives int64 triples
 * (after_item, grad-region byte offset, bytes) — one per contiguous span, in bucket
 * order; *n = number of triples (buf may be NULL).  Every rank derives the identical
 * list from the broadcast plan, so NCCL calls match across ranks. */
ts_status ts_plan_grad_buckets(const ts_plan_t* p, uint64_t bucket_bytes, int64_t* buf, uint64_t cap, uint64_t* n);
/* Plan blob for the data-parallel broadcast (rank 0 plans, every rank deserializes):
 * serialize writes *n bytes (buf NULL: size query; TS_ERR_ARG when cap < *n).  The blob
 * carries a fingerprint of the graph; deserialize returns TS_ERR_ARG for a blob of another
 * graph, a malformed one, or any entry ts_plan_set would reject (opt / p_num / dim / lead,
 * parameters not reside, an illegal D-CH channel chain) — nothing is adopted then. */
/* Per-kernel roofline of the plan's compute items: the sum over every F / B / R
 * micro-op of max(algorithmic FLOP / tensor_flops, algorithmic HBM bytes / hbm_bw), with the
 * same per-op FLOP and byte counts as the analytic profile (no launch or wave terms); also the
 * totals.  A lower bound on the step's compute-stream time on this plan. */
ts_status ts_plan_roofline(const ts_plan_t* p, double tensor_flops, double hbm_bw, double* seconds, double* flop,
                           double* bytes);
ts_status ts_plan_serialize(const ts_plan_t* p, void* buf, uint64_t cap, uint64_t* n);
ts_status ts_plan_deserialize(const ts_graph_t* g, const void* buf, uint64_t n, ts_plan_t** out);
void ts_plan_destroy(ts_plan_t* p);

/* ---- session (device) ---------------------------------------------------------- */
typedef struct {
  int32_t device;            /* CUDA ordinal                                          */
  void* slab;                /* device pointer lent by the caller (torch), >= bytes   */
  uint64_t slab_bytes;       /* the pool: static region + dynamic pool (= budget)     */
  void* stream_compute;      /* cudaStream_t or NULL (session creates its own)        */
  void* stream_d2h;
  void* stream_h2d;
  void* nccl_comm;           /* ncclComm_t for data-parallel allreduce, or NULL       */
  int32_t world_size;        /* gradient scale 1/world after the allreduce            */
  int32_t use_cuda_graph;    /* capture the whole step once and replay it             */
  float lr;                  /* SGD learning rate (0 = no update)                     */
  uint32_t step0;            /* dropout counter base                                  */
  int64_t sample_offset;     /* global index of this rank's first sample: dropout
                                counters (R15) use global sample indices, so the N ranks
                                of a data-parallel step draw disjoint masks and together
                                compute the step of the concatenated batch (0 on 1 GPU)   */
  int32_t host_numa_node;    /* NUMA node of the pinned swap pool: >= 0 that node, -1 the
                                GPU's own node (sysfs), -2 no binding (cudaHostAlloc)     */
  int32_t grad_allreduce_bf16; /* 1: each gradient bucket is rounded to bf16, summed by
                                ncclAllReduce in bf16 and widened back into the fp32
                                gradients (half the bytes on the link; the sum rounds to
                                bf16 — the fp32 masters and SGD stay fp32).  Needs a bf16
                                staging buffer of the largest bucket / 2 outside the slab.  0:
                                fp32 buckets                                                */
} ts_session_cfg;

/* Lays out the static region, allocates the pinned host swap pool, uploads
 * nothing (parameters start at zero until ts_set_param). */
ts_status ts_session_create(const ts_graph_t* g, const ts_plan_t* p, const ts_session_cfg* cfg,
                            ts_session_t** out);
void ts_session_destroy(ts_session_t* s);
/* Upload a parameter from host fp32 (count = numel); also refreshes its bf16 copy. */
ts_status ts_set_param(ts_session_t* s, int32_t tensor_id, const float* host_f32);
/* Download the fp32 master / fp32 gradient of a parameter to host. */
ts_status ts_get_param(ts_session_t* s, int32_t tensor_id, float* host_f32);
ts_status ts_get_grad(ts_session_t* s, int32_t tensor_id, float* host_f32);
ts_status ts_param_ptr(ts_session_t* s, int32_t tensor_id, void** dev_f32);
ts_status ts_grad_ptr(ts_session_t* s, int32_t tensor_id, void** dev_f32);
/* One training step: forward, backward, allreduce (if a comm is set), SGD.
 * inputs[i] = pointer to the i-th INPUT/LABEL tensor in tensor-id order
 * (int32 or the graph dtype), on the host if inputs_on_host != 0 (copied H2D
 * inside the step) else on the device (copied D2D).  Synchronous on return;
 * *loss_out = the global-batch mean loss of this rank's samples. */
ts_status ts_step(ts_session_t* s, const void* const* inputs, int32_t inputs_on_host, float* loss_out);
/* Same as ts_step but does not synchronise or read the loss back (bench loop). */
ts_status ts_step_async(ts_session_t* s, const void* const* inputs, int32_t inputs_on_host);
/* Allocation trace the runtime recorded on its last step (must equal ts_plan_trace). */
ts_status ts_session_trace(const ts_session_t* s, ts_alloc_event* buf, uint64_t cap, uint64_t* n);
/* The pinned host swap pool: bytes (= the plan's swapped bytes, 256-B slots) and the NUMA
 * node its pages are bound to (-1: unbound / unknown). */
ts_status ts_session_host_pool(const ts_session_t* s, uint64_t* bytes, int32_t* numa_node);
/* Kernel launches per step issued by the session (for gpu_launches accounting). */
ts_status ts_session_launches(const ts_session_t* s, int64_t* n);
/* Profiling (eager steps, cudaEvent pairs): enable / disable; then per item of the
 * augmented schedule (plan item order) the duration of its last execution in ms —
 * compute items on the compute stream, swap-out / swap-in copies on the D2H / H2D
 * stream (achieved PCIe bandwidth = piece bytes / copy time). */
ts_status ts_session_profile_items(ts_session_t* s, int32_t enable);
ts_status ts_session_item_times(const ts_session_t* s, float* ms, uint64_t cap, uint64_t* n);
/* Per-GEMM-launch records of the last profiled step: algorithmic FLOP (0 for the SIMT
 * fallback), cudaEvent duration on the compute stream (ms), batch count (1 = linear). */
ts_status ts_session_gemm_times(const ts_session_t* s, double* flop, float* ms, int32_t* batch, uint64_t cap,
                                uint64_t* n);
/* Kind of each record of ts_session_gemm_times: 0 GEMM (linear / attention), 1 conv
 * fprop, 2 conv dgrad, 3 conv wgrad (implicit GEMM); tc[i] = 1 when the tcgen05 path ran. */
ts_status ts_session_gemm_kinds(const ts_session_t* s, int32_t* kind, int32_t* tc, uint64_t cap, uint64_t* n);
/* Shape of each record: int32 quadruples (M, N, K, flags); flags bit0 A MN-major, bit1 B
 * MN-major, bit2 fp32 C, bit3 beta != 0 (GEMMs; convs report their implicit-GEMM M, N, K). */
ts_status ts_session_gemm_shapes(const ts_session_t* s, int32_t* mnkf, uint64_t cap, uint64_t* n);

/* ---- data parallelism (north_star: DP over NVLink with NCCL) -------------------
 * The session allreduces the fp32 gradient region (sum) with this communicator
 * on the compute stream after the backward pass, then scales by 1/world in SGD.
 * Bootstrap: rank 0 calls ts_nccl_unique_id (128 opaque bytes), the caller
 * broadcasts them (torch.distributed), every rank calls ts_nccl_comm_init.
 * NCCL is resolved from the libnccl.so.2 already in the process (torch's). */
ts_status ts_nccl_unique_id(void* out128);
ts_status ts_nccl_comm_init(const void* id128, int32_t nranks, int32_t rank, void** comm);
ts_status ts_nccl_comm_destroy(void* comm);

/* ---- kernels exposed for unit tests (device pointers, compute stream) -------- */
/* C[b] = alpha * op(A[b]) op(B[b]) (+ beta*C + bias): bf16 in, fp32 accumulate on
 * tcgen05 (TMEM), out bf16 or f32.  ta/tb = 1 when the operand's contiguous dim is
 * M (resp. N) rather than K.  Strides are in elements. */
ts_status ts_gemm_bf16(int32_t M, int32_t N, int32_t K, int32_t batch,
                       const void* A, int64_t lda, int64_t strideA, int32_t ta,
                       const void* B, int64_t ldb, int64_t strideB, int32_t tb,
                       void* C, int64_t ldc, int64_t strideC, int32_t c_dtype,
                       float alpha, float beta, const void* bias_bf16, void* stream);
/* Grouped product on the tcgen05 path (the session's q/k/v horizontal fusion), bf16
 * operands, device pointers, arrays of `groups` (<= 3) host-side pointers.  M, N, K
 * are TOTAL extents; a group spans 1/groups of the gdim extent:
 *   gdim 1 (N): C[g] = alpha A[0] op(B[g]) + bias[g] (+ beta C[g]), C[g] is M x N/groups
 *   gdim 2 (K): C[0] = alpha sum_g A[g] op(B[g]) + bias[0] (+ beta C[0]), A[g]: M x K/groups
 *   gdim 3 (M): C[g] = alpha A[g] op(B[0]) + bias[0] (+ beta C[g]), A[g]: M/groups x K
 * lda/ldb/ldc/ta/tb/c_dtype as in ts_gemm_bf16 (shared by all groups); beta 0 or 1;
 * bias may be NULL.  One grouped tcgen05 launch when a tiling fits (the tile must not
 * straddle groups: N/groups a multiple of 64, M/groups of 128, K/groups of 64), else the
 * groups run as plain products — the same values except for gdim 2 with a bf16 C, where
 * the per-group fallback rounds the running sum to bf16 after every group (the grouped
 * launch rounds once).  TS_ERR_ARG for bad groups / gdim, a grouped extent (N, K or M)
 * that `groups` does not divide, or beta other than 0 / 1. */
/* Fused-epilogue product (the session's linear -> gelu / gelu' peepholes, reading
 * D-FUSE), bf16 row-major operands as ts_gemm_bf16 with batch 1, bf16 C, beta 0:
 *   epi 1: C = U = alpha A op(B) + bias, aux = gelu(bf16(U))            (aux written)
 *   epi 2: C = dU = bf16(alpha A op(B)) * gelu'(aux), aux = U            (aux read)
 * aux is [M, N] row-major with leading dimension ldaux (elements).  TS_ERR_ARG for an
 * epi other than 1 / 2 or a shape / alignment the tcgen05 TMA-store path cannot take. */
ts_status ts_gemm_bf16_epi(int32_t epi, int32_t M, int32_t N, int32_t K, const void* A, int64_t lda, int32_t ta,
                           const void* B, int64_t ldb, int32_t tb, void* C, int64_t ldc, float alpha,
                           const void* bias_bf16, void* aux, int64_t ldaux, void* stream);
/* Row kernels for unit tests / microbenchmarks: op 0 = bias-gradient column sum,
 * out[j] (+)= sum_r x[r, j] over a [rows, n] row-major tensor (fp32 out; ws: device
 * workspace of ws_bytes >= 8 KB, its last 4 KB hold completion tickets that must start
 * zeroed).  `aux` unused.  Asynchronous on `stream`. */
ts_status ts_row_op(int32_t op, int32_t dtype, const void* x, const void* aux, void* out, int64_t rows, int32_t n,
                    float* ws, uint64_t ws_bytes, int32_t acc, void* stream);
ts_status ts_gemm_bf16_grouped(int32_t groups, int32_t gdim, int32_t M, int32_t N, int32_t K,
                               const void* const* A, int64_t lda, int32_t ta,
                               const void* const* B, int64_t ldb, int32_t tb,
                               void* const* C, int64_t ldc, int32_t c_dtype, float alpha, float beta,
                               const void* const* bias, void* stream);
/* Tile-selection override for the tcgen05 GEMM (tests and microbenchmarks; process-
 * wide, not thread-safe against concurrent launches): mode 0 = cost model (default),
 * 1 = single-CTA 128-row tiles only, 2 = CTA-pair (cta_group::2, 256-row) tiles
 * whenever M > 128 and N > 64; + 4 = never run the last partial wave as half-width
 * units.  TS_ERR_ARG for any other value. */
ts_status ts_gemm_set_mode(int32_t mode);
/* Configuration of the last tcgen05 GEMM launch: out8 = {tile width, CTAs per tile
 * (1 or 2), split-K factor, work units, SMs, co-resident CTA pairs, first half-width
 * tail unit (= work units when the tail wave is not split), 0}.  Host memory, 8 int32
 * written; TS_ERR_ARG when out8 is NULL. */
ts_status ts_gemm_last_config(int32_t* out8);
ts_status ts_gemm_f32(int32_t M, int32_t N, int32_t K,
                      const float* A, int64_t lda, int32_t ta,
                      const float* B, int64_t ldb, int32_t tb,
                      float* C, int64_t ldc, float alpha, float beta, const float* bias, void* stream);

/* Convolution micro-op kernels (unit tests; the session uses the same ones).
 * Cites: SURVEY.md §8(a) a6/a8 (C2/C3 conv as implicit GEMM), P:L260 (a micro-op
 * is a block of samples; dW merges by summation).  Layout: x [n,H,W,C] (NHWC),
 * w [K,R,S,C] (KRSC), y / dy [n,P,Q,K] with P = (H + 2 pad - R)/stride + 1 (same
 * for Q).  geom = {n, H, W, C, K, R, S, stride, pad}; all device pointers.
 *   mode 1 fprop: out = y (graph dtype) = conv(x, w) (+ bias[K], may be NULL)
 *   mode 2 dgrad: out = dx (graph dtype) (+)= conv_transpose(dy, w)   (acc != 0 adds)
 *   mode 3 wgrad: out = dw (fp32 [K,R,S,C]) (+)= sum over pixels of dy (x) im2col(x)
 * dtype TS_BF16: tcgen05/TMEM implicit GEMM with cp.async gathers (fp32 accumulate)
 * when eligible (K % 8 == 0; dgrad also C % 8 == 0), else CUDA cores; TS_F32: CUDA
 * cores with fp64 accumulation.  *used_tc (may be NULL) reports the path taken.
 * Layers with C % 64 == 0, K % 64 == 0 and stride <= 2 take the TMA-fed kernel
 * (spatial-box M tiles); mode | 0x10 forces the cp.async gather kernel (tests).
 * Errors: TS_ERR_ARG for bad geometry, TS_ERR_CUDA for launch failures. */
ts_status ts_conv2d(int32_t mode, int32_t dtype, const int32_t* geom, const void* x, const void* w, const void* dy,
                    void* out, const void* bias, int32_t acc, void* stream, int32_t* used_tc);

/* Fused attention micro-op kernels (unit tests; the session uses the same ones).
 * Cites: SURVEY.md §8(f) f2; semantics of TS_OP_ATTENTION above.  Q, K, V, C, dC, dQ,
 * dK, dV: device [nb*seq, heads*d] (row stride heads*d); lse: device fp32 [nb, heads, seq];
 * mask: device keep bits [nb, heads, seq, seq/32] (key j of a row at bit j%32; seq % 32 == 0),
 * written by the forward (may be NULL there), read by the backward;
 * ws: device fp32 scratch >= nb*heads*seq floats (backward).  geom = {nb, heads, seq, d,
 * dropout seed, b0 (global index of the first sample, for the dropout counters), step};
 * fattr = {alpha, p}.  mode 1: forward (writes C and lse; either may be NULL);
 * mode 2: backward (reads Q, K, V, C, lse, mask, dC; writes dQ, dK, dV, any may be NULL;
 * acc bit 0/1/2 adds into dQ/dK/dV).  mode | 0x10 forces the CUDA-core kernels.
 * dtype TS_BF16 with d = 64 and seq % 64 == 0 runs the tensor-core (mma.sync) kernels.
 * With seq % 128 == 0 and seq <= 512 the tcgen05 kernels run (*used_tc = 2) unless acc
 * bit 8 (0x100) asks for the mma.sync ones.
 * *used_tc reports the path (0 CUDA cores, 1 mma.sync, 2 tcgen05).  Errors: TS_ERR_ARG, TS_ERR_CUDA. */
ts_status ts_attention(int32_t mode, int32_t dtype, const int32_t* geom, const float* fattr, const void* q,
                       const void* k, const void* v, void* c, float* lse, uint32_t* mask, const void* dc, void* dq,
                       void* dk, void* dv, int32_t acc, float* ws, void* stream, int32_t* used_tc);

#ifdef __cplusplus
}
#endif
#endif
