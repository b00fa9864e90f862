// Host-side core of the TSPLIT runtime: graph, Alg. 1 schedule, augmented
// schedule expansion, best-fit pool simulation and the Alg. 2 planner.
// Semantics: DESIGN.md §4 (readings R1-R3, R10-R12 of SURVEY.md §8(c)).
#pragma once
#include <array>
#include <cstdint>
#include <string>
#include <unordered_map>
#include <vector>

#include "../../../include/ts.h"

namespace ts {

constexpr uint64_t kAlign = 256;
constexpr uint64_t kWsRows = 256;
constexpr uint64_t kInf = uint64_t(1) << 62;

inline uint64_t align_up(uint64_t n) { return (n + kAlign - 1) / kAlign * kAlign; }
// Ops whose statistics span the whole batch (R13): first micro-op reads every piece.
inline bool batch_reduce(int kind) { return kind == TS_OP_BATCHNORM; }
inline int dtype_bytes(int d) { return d == TS_BF16 ? 2 : 4; }
// Auxiliary outputs (statistics an op keeps for its own backward; no gradient): the
// fused attention's row log-sum-exp and dropout keep bits.
inline bool aux_output(int kind, int idx) { return kind == TS_OP_ATTENTION && (idx == 1 || idx == 2); }

void set_error(const std::string& msg);

struct Tensor {
  int id = 0, dtype = TS_F32, kind = TS_ACT, ndim = 0;
  int64_t shape[6] = {0, 0, 0, 0, 0, 0};
  int64_t numel = 0;
  uint64_t bytes = 0;
  bool sample = false;    // carries the split (sample) leading dim
  bool is_loss = false;
  bool needs_grad = false;
  int producer = -1;
  std::vector<int> consumers;  // op ids, ascending
  int64_t rows_per_sample = 0; // shape[0] / samples
  int64_t elems_per_sample = 0;
};

struct Op {
  int id = 0, kind = 0;
  std::vector<int> in, out;
  std::vector<int64_t> ia;
  std::vector<double> fa;
  bool has_bwd = false;
  std::vector<int> saved;  // non-param forward tensors the backward reads
};

struct Graph {
  int samples = 1, dtype = TS_F32;
  std::vector<Tensor> t;
  std::vector<Op> ops;
  std::vector<int> order;  // Alg. 1 forward schedule
  int loss = -1;
  // static region layout: masters | bf16 copies | grads | workspace
  std::vector<uint64_t> master_off, copy_off, grad_off;
  uint64_t ws_off = 0, ws_bytes = 0, static_bytes = 0;
  std::vector<uint64_t> bn_off;  // per op: [mean, rstd | sum dy*g, sum dy*g*xhat] fp32 (batch-stat ops)
  int n() const { return (int)t.size(); }
};

// Build + validate; returns TS_OK or an error with set_error().
ts_status build_graph(const ts_tensor_desc* td, int nt, const ts_op_desc* od, int no, int samples,
                      int dtype, Graph& g);

struct Cfg {
  int opt = TS_RESIDE, p = 1, dim = 0, lead = 1;
  int lag = 0;  // D-LAG: compute items after a swap-out before its range is reusable
};

// Piece = (key, j) with key = tensor id or n + id for the gradient of id.
using PieceKey = int64_t;
inline PieceKey pk(int key, int j) { return (int64_t(key) << 20) | int64_t(j); }
inline int pk_key(PieceKey p) { return int(p >> 20); }
inline int pk_j(PieceKey p) { return int(p & 0xFFFFF); }

enum ItemKind : int { IT_F = 0, IT_B = 1, IT_R = 2, IT_SO = 3, IT_SI = 4 };

struct Item {
  int kind = IT_F, op = -1, k = 0, group = -1;
  std::vector<PieceKey> reads, writes;
  std::vector<PieceKey> temps;  // D-ATTR staging temporaries (key 2n + op / 3n + op), live during the item
};

struct Expansion {
  std::vector<Item> items;
  std::vector<std::vector<PieceKey>> alloc_at;  // per item, ordered
  std::vector<std::vector<PieceKey>> free_after;
  int fwd_end = 0;
  std::vector<int> P;  // micro-op count per op
  std::unordered_map<PieceKey, uint64_t> temp_bytes;  // D-ATTR staging temporaries
  uint64_t bytes(const Graph& g, const std::vector<Cfg>& cfg, PieceKey pc) const;
};

// D-CH channel (parameter-dim) splits (expand.cpp)
bool is_chan(const Graph& g, const std::vector<Cfg>& cfg, int key);
bool channel_mode(const Graph& g, const std::vector<Cfg>& cfg, int op);
bool channel_ok(const Graph& g, const std::vector<Cfg>& cfg, std::string& why);
bool chan_local(const Graph& g, int op);  // maps channel block k to block k

// D-ATTR attribute (height / width) splits (expand.cpp; oracle/sim.py check_attr / staged_rect)
bool is_attr(const Graph& g, const std::vector<Cfg>& cfg, int key);
inline int attr_axis(const std::vector<Cfg>& cfg, int t) { return cfg[t].dim == 2 ? 1 : 2; }  // NHWC axis
bool attr_mode(const Graph& g, const std::vector<Cfg>& cfg, int op);   // an output is band-split
bool attr_window(int kind);                                              // conv2d / maxpool
bool attr_staged(const Graph& g, const std::vector<Cfg>& cfg, int op);  // window op reading / writing bands
bool attr_ok(const Graph& g, const std::vector<Cfg>& cfg, std::string& why);
struct Window {
  int R, stride, pad;  // window extent along the axis (conv: R rows / S columns), stride, pad
};
Window window_geom(const Graph& g, int op, int axis = 1);
struct Staged {
  int64_t rlo, hs, clo, ws, nb;  // input rows [rlo, rlo + hs) x columns [clo, clo + ws) (padding
                                 // included) of nb samples
};
// staged input of micro-op k (of P) of window op `op`: band mode stages what output band k
// reads along the band's axis (everything along the other) of every sample, sample mode (a
// full merge) everything of samples block k
Staged staged_rect(const Graph& g, const std::vector<Cfg>& cfg, int op, int k, int P);
uint64_t staged_bytes(const Graph& g, const std::vector<Cfg>& cfg, int op, int k, int P);

struct Event {
  int64_t seq;
  int item, kind, key, piece;
  uint64_t offset, bytes;
};

struct SimResult {
  std::vector<Event> trace;
  std::vector<uint64_t> top;   // per item: end of the highest live block after allocs
  std::vector<uint64_t> live;  // per item: dynamic live bytes after allocs
  uint64_t peak_live = 0, peak_extent = 0;
  uint64_t d2h = 0, h2d = 0;
  int64_t n_replay = 0, n_compute = 0;
  std::unordered_map<PieceKey, uint64_t> offset;  // placement of each piece (last)
  // R12 fences: for each item, the swap-out items whose logically freed range this
  // item's allocations overlap and that its stream (compute, or H2D for swap-ins) has
  // not yet waited for; the runtime waits on exactly these copy events.
  std::vector<std::vector<int>> wait_so;
};

int piece_count(const Graph& g, const std::vector<Cfg>& cfg, int key);
uint64_t piece_bytes(const Graph& g, const std::vector<Cfg>& cfg, int key);
// cache_bytes: D-LRU recompute cache limit (0 = memory-centric, Fig. 11)
void expand(const Graph& g, const std::vector<Cfg>& cfg, Expansion& ex, uint64_t cache_bytes = 0);
// capacity = kInf for planning; the runtime uses the slab size (identical trace if it fits).
bool simulate(const Graph& g, const std::vector<Cfg>& cfg, const Expansion& ex, uint64_t capacity,
              SimResult& r, std::vector<std::vector<std::pair<PieceKey, uint64_t>>>* placements = nullptr);

// Best-fit pool with the tail rule.
class Pool {
 public:
  void reset(uint64_t base, uint64_t capacity);
  bool alloc(uint64_t bytes, uint64_t* off);
  void release(uint64_t off, uint64_t bytes);
  uint64_t top() const;  // start of the tail block
  uint64_t extent() const { return extent_; }

 private:
  std::vector<std::pair<uint64_t, uint64_t>> free_;  // (offset, len) sorted
  uint64_t cap_ = 0, extent_ = 0;
};

// ---- data-parallel gradient buckets (dp.cpp) ----------------------------------
struct GradBucket {
  int after_item = -1;                                // allreduce once this item has run
  std::vector<std::pair<uint64_t, uint64_t>> spans;   // (grad-region offset, bytes), contiguous runs
};
std::vector<GradBucket> grad_buckets(const Graph& g, const Expansion& ex, uint64_t bucket_bytes);

// ---- profile + planner ------------------------------------------------------
struct OpCost {
  double flop_f = 0, flop_b = 0;    // whole op
  double bytes_f = 0, bytes_b = 0;  // algorithmic HBM bytes, whole op
  int kern_f = 1, kern_b = 1;       // kernels per micro-op
};
OpCost op_cost(const Graph& g, int op);

struct Profile {
  ts_hw hw;
  // time[op][log2 p] for fwd and bwd (whole op, all micro-ops)
  std::vector<std::array<double, 5>> tf, tb;
};
void profile_analytic(const Graph& g, const ts_hw& hw, Profile& pr);
ts_hw default_hw();

struct PlanState {
  std::vector<Cfg> cfg;
  uint64_t cache = 0;  // D-LRU recompute cache limit (bytes); 0 = memory-centric
  Expansion ex;
  SimResult sim;
  double predicted_s = 0, flop = 0;
};
void plan_refresh(const Graph& g, PlanState& ps, const Profile* pr);
ts_status plan_greedy(const Graph& g, uint64_t budget, const Profile& pr, PlanState& ps, uint32_t flags = 0);
// internal planner flag: Alg. 2 without D-LAG swap candidates (the post-pass may still add lags)
constexpr uint32_t kPlanNoLag = 1u << 30;
// Alg. 2 with D-LAG candidates, falling back to the run without them when that path dead-ends
// (lagged swaps hold their range for the copy; a later bottleneck inside the window can leave
// the greedy without candidates)
ts_status plan_greedy_lag(const Graph& g, uint64_t budget, const Profile& pr, PlanState& ps, uint32_t flags = 0);
void plan_refine(const Graph& g, uint64_t budget, const Profile& pr, PlanState& ps);
// D-LRU post-pass: the recompute cache limit the timeline predicts fastest within `budget`
void plan_lru(const Graph& g, uint64_t budget, const Profile& pr, PlanState& ps);

}  // namespace ts

