// Profiling-based planner (§IV-B/C, §V-B).
//   Eq. 1  min T + dT(C) s.t. M_i - dM(C) <= M
//   Eq. 2  dM_i[s_j, c] = size(s_j) for live non-I/O tensors
//   Eq. 3  swap stall, reading R5, Oc_u from a simulated
//                       PCIe timeline ("we keep an array to simulate")
//   Eqs. 4-5 (absent)   recompute cost, reading R6: per backward use, the time of the
//                       producer chain back to the nearest non-recomputed ancestor
//   Eq. 6  split cost, reading R7: (p-1) dT[micro, c] + dT_split(p, dim),
//                       dT_split = sum_k T(op on split k) - T(op); dM from
//                       re-simulation of the candidate
//   Alg. 2 (body lost — reading R8): at each bottleneck op, step 1
//                       best dT/dM over live non-I/O tensors x {swap, recompute};
//                       step 2 best over the op's own tensors x {opt} x p_num x dim;
//                       step 3 apply the better; fail when no candidate remains.
#include <algorithm>
#include <cmath>
#include <limits>
#include <cstdio>
#include <cstdlib>
#include <set>

#include "core.h"

namespace ts {

ts_hw default_hw() {
  ts_hw hw;
  hw.tensor_flops = 1.3868e15;  // MEASURED_PEAKS bf16_tflops_sustained
  hw.simt_flops = 60e12;
  hw.hbm_bw = 6.55e12;          // MEASURED_PEAKS hbm_gbs
  hw.d2h_bw = 50e9;
  hw.h2d_bw = 50e9;
  hw.launch_s = 2.5e-6;
  return hw;
}

OpCost op_cost(const Graph& g, int oi) {
  const Op& o = g.ops[oi];
  OpCost c;
  double es = dtype_bytes(g.dtype);
  auto nb = [&](int t) { return double(g.t[t].numel) * es; };
  switch (o.kind) {
    case TS_OP_LINEAR: {
      double R = g.t[o.in[0]].shape[0], K = g.t[o.in[0]].shape[1], N = g.t[o.in[1]].shape[0];
      c.flop_f = 2 * R * N * K;
      c.flop_b = 4 * R * N * K;
      c.bytes_f = (R * K + N * K + R * N) * es;
      c.bytes_b = (2 * R * N + N * K + 2 * R * K) * es + 8 * N * K + 4 * R * N;
      c.kern_f = 1;
      c.kern_b = 3;
      break;
    }
    case TS_OP_ATTN_QK: case TS_OP_ATTN_PV: {
      const Tensor& s = g.t[o.kind == TS_OP_ATTN_QK ? o.out[0] : o.in[0]];
      const Tensor& q = g.t[o.kind == TS_OP_ATTN_QK ? o.in[0] : o.in[1]];
      double d = double(q.shape[1]) / double(o.ia[0]);
      c.flop_f = 2.0 * double(s.numel) * d;
      c.flop_b = 2 * c.flop_f;
      c.bytes_f = (2.0 * q.numel + s.numel) * es;
      c.bytes_b = (4.0 * q.numel + 2.0 * s.numel) * es;
      c.kern_b = 2;
      break;
    }
    case TS_OP_EMBED:
      c.bytes_f = 3 * nb(o.out[0]);
      c.bytes_b = 2 * nb(o.out[0]) + 8.0 * g.t[o.out[0]].numel;
      c.kern_b = 2;
      break;
    case TS_OP_LAYERNORM:
      c.bytes_f = 2 * nb(o.in[0]);
      c.bytes_b = 3 * nb(o.in[0]);
      c.kern_b = 2;
      break;
    case TS_OP_ADD:
      c.bytes_f = 3 * nb(o.out[0]);
      c.bytes_b = 3 * nb(o.out[0]);
      break;
    case TS_OP_XENT:
      c.bytes_f = 2 * nb(o.in[0]);
      c.bytes_b = 2 * nb(o.in[0]);
      break;
    case TS_OP_ATTENTION: {
      // fused: 2 products forward (S = QK^T, C = PV), 7 backward (dQ kernel: S, dP, dQ;
      // dK/dV kernel: S, dP, dV, dK); no [b,a,s,s] tensor touches HBM
      const Tensor& q = g.t[o.in[0]];
      const double heads = double(o.ia[0]), seq = double(o.ia[1]);
      const double d = double(q.shape[1]) / heads, nbt = double(q.shape[0]) / seq;
      const double unit = 2.0 * nbt * heads * seq * seq * d;
      c.flop_f = 2 * unit;
      c.flop_b = 7 * unit;
      c.bytes_f = 4 * nb(o.in[0]) + double(g.t[o.out[1]].bytes + g.t[o.out[2]].bytes);
      c.bytes_b = 8 * nb(o.in[0]) + 2.0 * double(g.t[o.out[1]].bytes + g.t[o.out[2]].bytes);
      c.kern_b = 3;
      break;
    }
    case TS_OP_CONV2D: {
      const Tensor &w = g.t[o.in[1]], &y = g.t[o.out[0]];
      const double rsc = double(w.shape[1]) * w.shape[2] * w.shape[3];
      c.flop_f = 2.0 * double(y.numel) * rsc;
      c.flop_b = 2 * c.flop_f;
      c.bytes_f = nb(o.in[0]) + nb(o.out[0]) + double(w.numel) * es;
      c.bytes_b = 2 * nb(o.in[0]) + 2 * nb(o.out[0]) + 8.0 * w.numel;
      c.kern_b = 2;
      break;
    }
    case TS_OP_BATCHNORM:
      c.bytes_f = 3 * nb(o.in[0]);
      c.bytes_b = 5 * nb(o.in[0]);
      c.kern_f = 2;
      c.kern_b = 2;
      break;
    default:  // elementwise / row ops
      c.bytes_f = nb(o.in[0]) + nb(o.out[0]);
      c.bytes_b = 3 * nb(o.out[0]);
      break;
  }
  return c;
}

namespace {
int lg2(int p) {
  int l = 0;
  while ((1 << l) < p) ++l;
  return std::min(l, 4);
}

// GEMM wave efficiency on 148 SMs with 128x256 tiles (the Fig. 5 effect).
double wave_eff(double M, double N, double batch) {
  double tiles = std::ceil(M / 128.0) * std::ceil(N / 256.0) * batch;
  if (tiles <= 0) return 1.0;
  double waves = std::ceil(tiles / 148.0);
  return tiles / (waves * 148.0);
}
}  // namespace

void profile_analytic(const Graph& g, const ts_hw& hw, Profile& pr) {
  pr.hw = hw;
  pr.tf.assign(g.ops.size(), {});
  pr.tb.assign(g.ops.size(), {});
  for (auto& o : g.ops) {
    OpCost c = op_cost(g, o.id);
    double peak = g.dtype == TS_BF16 ? hw.tensor_flops : hw.simt_flops;
    for (int l = 0; l < 5; ++l) {
      double p = double(1 << l);
      double eff = 1.0;
      if (o.kind == TS_OP_LINEAR)
        eff = wave_eff(g.t[o.in[0]].shape[0] / p, g.t[o.in[1]].shape[0], 1);
      else if (o.kind == TS_OP_ATTN_QK || o.kind == TS_OP_ATTN_PV) {
        const Tensor& s = g.t[o.kind == TS_OP_ATTN_QK ? o.out[0] : o.in[0]];
        double nbh = double(s.shape[0]) * s.shape[1] / p;
        eff = wave_eff(s.shape[2], o.kind == TS_OP_ATTN_QK ? s.shape[3] : 64, nbh);
      }
      eff = std::max(eff, 0.05);
      double tf = std::max(c.flop_f / p / (peak * eff), c.bytes_f / p / hw.hbm_bw);
      double tb = std::max(c.flop_b / p / (peak * eff), c.bytes_b / p / hw.hbm_bw);
      pr.tf[o.id][l] = p * (c.kern_f * hw.launch_s + tf);
      pr.tb[o.id][l] = p * (c.kern_b * hw.launch_s + tb);
    }
  }
}

namespace {

// Per-item time and the PCIe occupancy arrays (Oc_u) of the simulated timeline.
struct Timeline {
  std::vector<double> T, oc_d2h, oc_h2d;
  double total = 0;
};

void timeline(const Graph& g, const PlanState& ps, const Profile& pr, Timeline& tl) {
  const auto& items = ps.ex.items;
  size_t ni = items.size();
  tl.T.assign(ni, 0);
  tl.oc_d2h.assign(ni, 0);
  tl.oc_h2d.assign(ni, 0);
  std::vector<double> start(ni, 0);
  std::vector<std::pair<double, double>> busy_d2h, busy_h2d;
  std::unordered_map<PieceKey, double> ready, so_end;
  std::unordered_map<size_t, double> so_end_item;  // SO item -> copy completion time
  double clock = 0, d2h_free = 0, h2d_free = 0;
  for (size_t i = 0; i < ni; ++i) {
    const Item& it = items[i];
    if (it.kind == IT_SO) {
      double s = std::max(clock, d2h_free);
      so_end_item[i] = 0;
      double e = s + double(piece_bytes(g, ps.cfg, pk_key(it.reads[0]))) / pr.hw.d2h_bw;
      busy_d2h.push_back({s, e});
      d2h_free = e;
      so_end[it.reads[0]] = e;
      so_end_item[i] = e;
      continue;
    }
    if (it.kind == IT_SI) {
      double s = std::max(clock, h2d_free);
      auto so = so_end.find(it.writes[0]);
      if (so != so_end.end()) s = std::max(s, so->second);
      for (int f : ps.sim.wait_so[i]) s = std::max(s, so_end_item[size_t(f)]);
      double e = s + double(piece_bytes(g, ps.cfg, pk_key(it.writes[0]))) / pr.hw.h2d_bw;
      busy_h2d.push_back({s, e});
      h2d_free = e;
      ready[it.writes[0]] = e;
      continue;
    }
    for (PieceKey p : it.reads) {
      auto r = ready.find(p);
      if (r != ready.end()) clock = std::max(clock, r->second);
    }
    // reuse of a range still being copied out waits for that copy (R12)
    for (int f : ps.sim.wait_so[i]) clock = std::max(clock, so_end_item[size_t(f)]);
    int l = lg2(ps.ex.P[it.op]);
    double t = (it.kind == IT_B ? pr.tb[it.op][l] : pr.tf[it.op][l]) / double(ps.ex.P[it.op]);
    if (!it.temps.empty()) {  // D-ATTR staging: gather (read + write the staged rows), and in the
                              // backward the scatter-add (read the staged gradient, read + write dX)
      const double b = double(ps.ex.temp_bytes.at(it.temps[0]));
      t += it.kind == IT_B ? 2 * pr.hw.launch_s + 5 * b / pr.hw.hbm_bw : pr.hw.launch_s + 2 * b / pr.hw.hbm_bw;
    }
    start[i] = clock;
    tl.T[i] = t;
    clock += t;
  }
  // the step ends when the last transfer has drained too
  tl.total = std::max(clock, std::max(d2h_free, h2d_free));
  auto occ = [&](const std::vector<std::pair<double, double>>& busy, std::vector<double>& oc) {
    size_t b = 0;
    for (size_t i = 0; i < ni; ++i) {
      if (tl.T[i] <= 0) continue;
      double s = start[i], e = s + tl.T[i], cov = 0;
      while (b < busy.size() && busy[b].second <= s) ++b;
      for (size_t k = b; k < busy.size() && busy[k].first < e; ++k)
        cov += std::max(0.0, std::min(e, busy[k].second) - std::max(s, busy[k].first));
      oc[i] = std::min(1.0, cov / tl.T[i]);
    }
  };
  occ(busy_d2h, tl.oc_d2h);
  occ(busy_h2d, tl.oc_h2d);
}

// D-LAG release lag for swapping t in plan ps: the number of compute items after t's last
// forward toucher whose timeline time covers the D2H copy of all its bytes (+25 %).
int release_lag(const Graph& g, const PlanState& ps, const Timeline& tl, const Profile& pr, int t) {
  const auto& items = ps.ex.items;
  int last_fw = -1;
  for (int i = 0; i < ps.ex.fwd_end && i < (int)items.size(); ++i) {
    const Item& it = items[i];
    if (it.kind == IT_SO || it.kind == IT_SI) continue;
    for (PieceKey p : it.reads)
      if (pk_key(p) == t) last_fw = i;
    for (PieceKey p : it.writes)
      if (pk_key(p) == t) last_fw = i;
  }
  if (last_fw < 0) return 0;
  const double need = 1.25 * double(g.t[t].bytes) / pr.hw.d2h_bw;
  double acc_t = 0;
  int lag = 0;
  for (size_t u = size_t(last_fw) + 1; u < items.size() && acc_t < need && lag < 4096; ++u) {
    if (items[u].kind == IT_SO || items[u].kind == IT_SI) continue;
    acc_t += tl.T[u];
    ++lag;
  }
  return lag;
}

double flops_of(const Graph& g, const PlanState& ps) {
  double f = 0;
  for (auto& it : ps.ex.items) {
    if (it.kind == IT_SO || it.kind == IT_SI) continue;
    OpCost c = op_cost(g, it.op);
    f += (it.kind == IT_B ? c.flop_b : c.flop_f) / double(ps.ex.P[it.op]);
  }
  return f;
}

}  // namespace

void plan_refresh(const Graph& g, PlanState& ps, const Profile* pr) {
  expand(g, ps.cfg, ps.ex, ps.cache);
  simulate(g, ps.cfg, ps.ex, kInf, ps.sim);
  ps.flop = flops_of(g, ps);
  if (pr) {
    Timeline tl;
    timeline(g, ps, *pr, tl);
    ps.predicted_s = tl.total;
  }
}

namespace {

struct Cand {
  double ratio = std::numeric_limits<double>::infinity();
  int tensor = -1, opt = 0, p = 1, birth = 0;
  bool valid = false;
};

bool better(const Cand& a, const Cand& b) {  // a strictly better than b
  if (!b.valid) return a.valid;
  if (!a.valid) return false;
  if (a.ratio != b.ratio) return a.ratio < b.ratio;
  if (a.birth != b.birth) return a.birth < b.birth;  // earlier generated first
  return a.tensor < b.tensor;
}

}  // namespace

namespace {
uint64_t max_top(const PlanState& s) {
  uint64_t m = 0;
  for (uint64_t t : s.sim.top) m = std::max(m, t);
  return m;
}
}  // namespace

// Post-pass on the greedy plan (reading D-R8c).  Alg. 2 resolves bottlenecks
// in schedule order, so an eviction chosen at an early bottleneck can become redundant
// once later ones are fixed, and several prefetches can collide on the H2D link.
// (1) revert non-reside decisions, most expensive first, whenever the plan still fits;
// (2) turn remaining recomputes into swaps with longer prefetch leads when that lowers
// the predicted step time and still fits.  Every change is re-simulated.
void plan_refine(const Graph& g, uint64_t budget, const Profile& pr, PlanState& ps) {
  plan_refresh(g, ps, &pr);
  const int n = g.n();
  auto try_cfg = [&](const std::vector<Cfg>& cfg, PlanState& out) {
    std::string why;
    if (!channel_ok(g, cfg, why) || !attr_ok(g, cfg, why)) return false;  // e.g. reverting one block of a D-CH chain
    out.cfg = cfg;
    out.cache = ps.cache;
    plan_refresh(g, out, &pr);
    return max_top(out) <= budget;
  };
  // cost of each decision: predicted time saved by reverting it (ignoring feasibility)
  std::vector<std::pair<double, int>> order;
  for (int t = 0; t < n; ++t) {
    const Cfg& c = ps.cfg[t];
    if (c.opt == TS_RESIDE && c.p == 1) continue;
    PlanState tmp;
    std::vector<Cfg> cfg = ps.cfg;
    cfg[t] = Cfg();
    tmp.cfg = cfg;
    tmp.cache = ps.cache;
    plan_refresh(g, tmp, &pr);
    order.push_back({ps.predicted_s - tmp.predicted_s, t});
  }
  std::sort(order.begin(), order.end(), [](auto& a, auto& b) { return a.first > b.first; });
  for (auto& [gain, t] : order) {
    if (gain <= 0) continue;
    std::vector<Cfg> cfg = ps.cfg;
    cfg[t] = Cfg();
    PlanState cand;
    if (try_cfg(cfg, cand) && cand.predicted_s < ps.predicted_s) ps = std::move(cand);
  }
  // swaps whose freed range is reused while the copy still runs: release it later (D-LAG)
  for (int t = 0; t < n; ++t) {
    if (ps.cfg[t].opt != TS_SWAP || ps.cfg[t].lag > 0) continue;
    Timeline tl;
    timeline(g, ps, pr, tl);
    const int lag = release_lag(g, ps, tl, pr, t);
    if (lag <= 0) continue;
    std::vector<Cfg> cfg = ps.cfg;
    cfg[t].lag = lag;
    PlanState cand;
    if (try_cfg(cfg, cand) && cand.predicted_s < ps.predicted_s - 1e-6) ps = std::move(cand);
  }
  // recompute -> swap with a prefetch lead that hides the copy behind compute, and the
  // range released only after the copy (D-LAG)
  std::vector<std::pair<double, int>> rc;
  for (int t = 0; t < n; ++t)
    if (ps.cfg[t].opt == TS_RECOMPUTE) rc.push_back({double(g.t[t].bytes), t});
  std::sort(rc.begin(), rc.end(), [](auto& a, auto& b) { return a.first > b.first; });
  for (auto& [bytes, t] : rc) {
    (void)bytes;
    Timeline tl;
    timeline(g, ps, pr, tl);
    const int lag = release_lag(g, ps, tl, pr, t);
    bool done = false;
    for (int lead : {4, 16, 64}) {
      for (int lg : {lag, 0}) {
        std::vector<Cfg> cfg = ps.cfg;
        cfg[t].opt = TS_SWAP;
        cfg[t].lead = lead;
        cfg[t].lag = lg;
        PlanState cand;
        if (try_cfg(cfg, cand) && cand.predicted_s < ps.predicted_s - 1e-6) {
          ps = std::move(cand);
          done = true;
          break;
        }
        if (lag == 0) break;
      }
      if (done) break;
    }
  }
}

// LRU-based recomputation (reading D-LRU): the greedy plan is made memory-centric;
// then the recompute cache limit is chosen as the fastest feasible of {unbounded, the
// plan's headroom x 8, x 4, x 2, x 1, x 1/2} (headroom = budget - simulated peak, so the
// cached pieces only use memory the memory-centric plan leaves free), and with a cache the
// D-R8c post-pass runs again (decisions that no longer pay can be reverted).
// (plus rbytes / 2^k down to 1 MiB: the plan's peak is usually set in the forward pass, so a
// cache far larger than the headroom can still fit the backward)
void plan_lru(const Graph& g, uint64_t budget, const Profile& pr, PlanState& ps) {
  bool any = false;
  for (const Cfg& c : ps.cfg) any |= c.opt == TS_RECOMPUTE;
  if (!any) return;
  const uint64_t head = budget > max_top(ps) ? budget - max_top(ps) : 0;
  uint64_t rbytes = 0;  // every recompute-opt tensor: an upper bound on what can be cached
  for (int t = 0; t < g.n(); ++t)
    if (ps.cfg[t].opt == TS_RECOMPUTE) rbytes += g.t[t].bytes;
  PlanState best = ps;
  std::vector<uint64_t> caps = {~uint64_t(0), 8 * head, 4 * head, 2 * head, head, head / 2};
  for (uint64_t c = rbytes / 2; c > (uint64_t(1) << 20) && caps.size() < 24; c /= 2) caps.push_back(c);
  for (uint64_t cap : caps) {
    if (cap == 0) continue;
    PlanState cand;
    cand.cfg = ps.cfg;
    cand.cache = cap;
    plan_refresh(g, cand, &pr);
    if (max_top(cand) <= budget && cand.predicted_s < best.predicted_s - 1e-9) best = std::move(cand);
  }
  if (best.cache != ps.cache) {
    ps = std::move(best);
    plan_refine(g, budget, pr, ps);
  }
}

ts_status plan_greedy(const Graph& g, uint64_t budget, const Profile& pr, PlanState& ps, uint32_t flags) {
  const int n = g.n();
  ps.cfg.assign(n, Cfg());
  if (g.static_bytes > budget) {
    set_error("budget below the static region (" + std::to_string(g.static_bytes) + " B)");
    return TS_ERR_INFEASIBLE;
  }
  std::vector<int> birth(n, 0);
  for (size_t i = 0; i < g.order.size(); ++i)
    for (int x : g.ops[g.order[i]].out) birth[x] = (int)i;
  const int kMaxIter = 20000;
  for (int iter = 0; iter < kMaxIter; ++iter) {
    plan_refresh(g, ps, &pr);
    const auto& items = ps.ex.items;
    int bi = -1;
    for (size_t i = 0; i < items.size(); ++i)
      if (ps.sim.top[i] > budget) {
        bi = (int)i;
        break;
      }
    if (bi < 0) {
      plan_refine(g, budget, pr, ps);
      if (!(flags & TS_PLAN_MEMORY_CENTRIC)) plan_lru(g, budget, pr, ps);
      return TS_OK;
    }
    // bottleneck op and phase
    int ci = bi;
    while (ci < (int)items.size() && (items[ci].kind == IT_SO || items[ci].kind == IT_SI)) ++ci;
    if (ci >= (int)items.size()) ci = bi - 1;
    while (ci >= 0 && (items[ci].kind == IT_SO || items[ci].kind == IT_SI)) --ci;
    if (ci < 0) return set_error("no compute item near the bottleneck"), TS_ERR_INFEASIBLE;
    int bop = items[ci].op;
    bool bwd_phase = ci >= ps.ex.fwd_end;
    if (bwd_phase && items[ci].kind == IT_R) {
      for (int j = ci; j < (int)items.size(); ++j)
        if (items[j].kind == IT_B && items[j].group == items[ci].group) {
          bop = items[j].op;
          break;
        }
    }
    Timeline tl;
    timeline(g, ps, pr, tl);
    // per-tensor touch summary of the current expansion
    std::vector<int> last_fw(n, -1), first_bw(n, -1);
    std::vector<std::set<int>> bw_ops(n);
    for (size_t i = 0; i < items.size(); ++i) {
      const Item& it = items[i];
      if (it.kind == IT_SO || it.kind == IT_SI) continue;
      auto touch = [&](PieceKey p) {
        int key = pk_key(p);
        if (key >= n) return;
        if ((int)i < ps.ex.fwd_end) last_fw[key] = (int)i;
        else {
          if (first_bw[key] < 0) first_bw[key] = (int)i;
          int gop = it.op;
          if (it.kind == IT_R)
            for (size_t j = i; j < items.size(); ++j)
              if (items[j].kind == IT_B && items[j].group == it.group) {
                gop = items[j].op;
                break;
              }
          bw_ops[key].insert(gop);
        }
      };
      for (PieceKey p : it.reads) touch(p);
      for (PieceKey p : it.writes) touch(p);
    }
    // tensors touched by the bottleneck op in this phase
    std::set<int> own;
    for (size_t i = 0; i < items.size(); ++i) {
      bool same_phase = ((int)i >= ps.ex.fwd_end) == bwd_phase;
      if (!same_phase || items[i].op != bop) continue;
      for (PieceKey p : items[i].reads) own.insert(pk_key(p) % n);
      for (PieceKey p : items[i].writes) own.insert(pk_key(p) % n);
    }
    for (int x : g.ops[bop].in) own.insert(x);
    for (int x : g.ops[bop].out) own.insert(x);
    // live pieces at the bottleneck item
    std::set<int> live;
    {
      std::unordered_map<PieceKey, int> alive;
      for (auto& e : ps.sim.trace) {
        if (e.item > bi) break;
        PieceKey p = pk(e.key, e.piece);
        if (e.kind == 0) alive[p] = 1;
        else if (e.item < bi) alive.erase(p);
      }
      for (auto& kv : alive)
        if (pk_key(kv.first) < n) live.insert(pk_key(kv.first));
    }
    auto rc_time = [&](auto&& self, int t, int depth) -> double {
      const Tensor& x = g.t[t];
      if (x.kind != TS_ACT || depth > 64) return 0.0;
      int po = x.producer;
      double tm = pr.tf[po][lg2(ps.ex.P[po])];
      for (int u : g.ops[po].in)
        if (g.t[u].kind == TS_ACT && ps.cfg[u].opt == TS_RECOMPUTE) tm += self(self, u, depth + 1);
      return tm;
    };
    auto swap_cost = [&](int t, double size) {
      int j = last_fw[t], q = first_bw[t];
      if (j < 0 || q < 0) return std::numeric_limits<double>::infinity();
      int p = std::max(q - std::max(1, ps.cfg[t].lead), ps.ex.fwd_end);
      double fw = 0, bw = 0;
      for (int u = j + 1; u < bi && u < (int)items.size(); ++u) fw += (1.0 - tl.oc_d2h[u]) * tl.T[u];
      for (int u = p; u < q; ++u) bw += (1.0 - tl.oc_h2d[u]) * tl.T[u];
      return std::max(0.0, size / pr.hw.d2h_bw - fw) + std::max(0.0, size / pr.hw.h2d_bw - bw);
    };
    // D-LAG: compute items after t's swap-out whose profiled time covers the copy of all its
    // pieces at the D2H bandwidth (+25 %), so the freed range is reused after the copy ends
    auto lag_for = [&](int t) -> int {
      if (last_fw[t] < 0 || (flags & kPlanNoLag)) return 0;
      const double need = 1.25 * double(g.t[t].bytes) / pr.hw.d2h_bw;
      double acc_t = 0;
      int lag = 0;
      for (size_t u = size_t(last_fw[t]) + 1; u < items.size() && acc_t < need && lag < 4096; ++u) {
        if (items[u].kind == IT_SO || items[u].kind == IT_SI) continue;
        acc_t += tl.T[u];
        ++lag;
      }
      return lag;
    };
    // ---- candidates ---------------------------------------------------------------
    struct Change {
      int t, opt, p, lead, dim = -1;  // dim -1: keep the tensor's split dim
      int lag = 0;                    // D-LAG release lag (swap only)
    };
    struct Cand2 {
      std::vector<Change> ch;
      double analytic = 0;
      int birth = 0, tensor = 0;
    };
    // recompute of t also recomputes producer inputs that would otherwise be held only
    // for the replay (e.g. attention scores behind a recomputed softmax output)
    auto with_feeders = [&](Cand2 c, int t) {
      const Op& po = g.ops[g.t[t].producer];
      for (int u : po.in) {
        const Tensor& x = g.t[u];
        if (x.kind == TS_ACT && !x.is_loss && u != t && ps.cfg[u].opt == TS_RESIDE && first_bw[u] < 0)
          c.ch.push_back({u, TS_RECOMPUTE, ps.cfg[u].p, 1});
      }
      return c;
    };
    std::vector<Cand2> step1, step2;
    // step 1: non-split options on live tensors that are neither inputs nor outputs of
    // the bottleneck op (Eq. 2 dM, Eq. 3 / R6 dT for the shortlist)
    for (int t : live) {
      const Tensor& x = g.t[t];
      if (x.kind != TS_ACT || x.is_loss || ps.cfg[t].opt != TS_RESIDE || own.count(t)) continue;
      if (first_bw[t] < 0) continue;                 // not held for backward: nothing to gain
      if (!bwd_phase && last_fw[t] >= bi) continue;  // still read later in the forward pass
      if (bwd_phase && first_bw[t] <= bi) continue;  // read by the bottleneck or before it
      double dm = double(x.bytes);
      Cand2 c;
      c.birth = birth[t];
      c.tensor = t;
      // a recompute replays in the group of the first backward reader, after the bottleneck,
      // so it frees t there even when that reader is the very next item; a swap-in lands
      // `lead` compute items earlier, so it frees t only when that is still after bi
      if (bwd_phase && first_bw[t] - std::max(1, ps.cfg[t].lead) <= bi) {
        c.ch = {{t, TS_RECOMPUTE, ps.cfg[t].p, 1}};
        c.analytic = double(bw_ops[t].size()) * rc_time(rc_time, t, 0) / dm;
        step1.push_back(with_feeders(c, t));
        continue;
      }
      c.ch = {{t, TS_SWAP, ps.cfg[t].p, 1}};
      c.analytic = swap_cost(t, dm) / dm;
      step1.push_back(c);
      const int lag = lag_for(t);
      if (lag > 0) {  // the same swap with its range released after the copy (D-LAG)
        Cand2 cl = c;
        cl.ch[0].lag = lag;
        step1.push_back(cl);
      }
      // the same swap with the prefetch issued early enough to hide the H2D copy
      // (B200 computes ~30x more per PCIe byte than the paper's GPUs)
      {
        double need = 1.25 * dm / pr.hw.h2d_bw, acc_t = 0;
        int lead = 0;
        for (int u = first_bw[t] - 1; u >= ps.ex.fwd_end && acc_t < need; --u) {
          if (items[u].kind == IT_SO || items[u].kind == IT_SI) continue;
          acc_t += tl.T[u];
          ++lead;
        }
        if (lead > 1) {
          Cand2 c2 = c;
          c2.ch = {{t, TS_SWAP, ps.cfg[t].p, lead}};
          double fw = 0;
          for (int u = last_fw[t] + 1; u < bi && u < (int)items.size(); ++u) fw += (1.0 - tl.oc_d2h[u]) * tl.T[u];
          c2.analytic = std::max(0.0, dm / pr.hw.d2h_bw - fw) / dm;
          step1.push_back(c2);
          if (lag > 0) {
            Cand2 c3 = c2;
            c3.ch[0].lag = lag;
            c3.analytic = 0.0;  // both copies hidden behind profiled compute
            step1.push_back(c3);
          }
        }
      }
      c.ch = {{t, TS_RECOMPUTE, ps.cfg[t].p, 1}};
      c.analytic = double(bw_ops[t].size()) * rc_time(rc_time, t, 0) / dm;
      step1.push_back(with_feeders(c, t));
    }
    // a swapped tensor live at a backward bottleneck only because its prefetch lands early
    // (long lead): shorten the lead to the previous computation or recompute it
    if (bwd_phase)
      for (int t : live) {
        const Tensor& x = g.t[t];
        if (x.kind != TS_ACT || x.is_loss || ps.cfg[t].opt != TS_SWAP || own.count(t)) continue;
        if (first_bw[t] <= bi) continue;
        const double dm = double(x.bytes);
        Cand2 c;
        c.birth = birth[t];
        c.tensor = t;
        if (ps.cfg[t].lead > 1) {
          c.ch = {{t, TS_SWAP, ps.cfg[t].p, 1}};
          c.analytic = swap_cost(t, dm) / dm;
          step1.push_back(c);
        }
        c.ch = {{t, TS_RECOMPUTE, ps.cfg[t].p, 1}};
        c.analytic = double(bw_ops[t].size()) * rc_time(rc_time, t, 0) / dm;
        step1.push_back(with_feeders(c, t));
      }
    // shortlist by the analytic ratio, keeping the best swaps and the best recomputes
    {
      auto by = [](const Cand2& a, const Cand2& b) {
        if (a.analytic != b.analytic) return a.analytic < b.analytic;
        return a.birth < b.birth;
      };
      std::vector<Cand2> sw, rc;
      for (auto& c : step1) (c.ch[0].opt == TS_SWAP ? sw : rc).push_back(c);
      std::stable_sort(sw.begin(), sw.end(), by);
      std::stable_sort(rc.begin(), rc.end(), by);
      if (sw.size() > 10) sw.resize(10);
      if (rc.size() > 8) rc.resize(8);
      step1 = sw;
      step1.insert(step1.end(), rc.begin(), rc.end());
    }
    // step 2: split options on the bottleneck op's own activations (Eq. 6); the
    // "TSPLIT w/o Split" ablation of P:L463 plans with steps 1 and 3 only
    const bool no_split = flags & TS_PLAN_NO_SPLIT;
    std::vector<int> split_cands;
    for (int x : g.ops[bop].in)
      if (g.t[x].kind == TS_ACT && !g.t[x].is_loss) split_cands.push_back(x);
    for (int x : g.ops[bop].out)
      if (g.t[x].kind == TS_ACT && !g.t[x].is_loss) split_cands.push_back(x);
    for (int t : split_cands)
      for (int p = 2; p <= 16 && !no_split; p *= 2) {
        if (p <= ps.cfg[t].p || g.samples % p) continue;
        for (int opt : {TS_RESIDE, TS_SWAP, TS_RECOMPUTE}) {
          if (opt != TS_RESIDE && first_bw[t] < 0) continue;
          Cand2 c;
          c.birth = birth[t];
          c.tensor = t;
          c.ch = {{t, opt, p, ps.cfg[t].lead}};
          step2.push_back(opt == TS_RECOMPUTE ? with_feeders(c, t) : c);
          if (opt == TS_SWAP && lag_for(t) > 0) {  // D-LAG variant
            c.ch[0].lag = lag_for(t);
            step2.push_back(c);
          }
        }
      }
    // D-CH: channel (parameter-dim) splits of the bottleneck op's 2-D activations, with the
    // elementwise neighbours that must share the blocks (linear -> gelu -> linear: the
    // FFN's [T, 4h] pair); illegal combinations are dropped by channel_ok in consider()
    auto ew = [&](int kind) { return kind == TS_OP_RELU || kind == TS_OP_GELU || kind == TS_OP_TANH; };
    for (int t : split_cands) {
      const Tensor& x = g.t[t];
      if (no_split || x.ndim != 2 || first_bw[t] < 0 || is_chan(g, ps.cfg, t)) continue;
      // only once the sample dim is exhausted (Fig. 6: the sample split is bounded by the
      // batch — small-batch / large-model training is where the parameter dim pays)
      bool sample_room = false;
      for (int p = 2 * ps.cfg[t].p; p <= 16; p *= 2) sample_room |= g.samples % p == 0;
      if (sample_room) continue;
      std::vector<int> chain{t};
      for (int u = t; g.t[u].producer >= 0 && ew(g.ops[g.t[u].producer].kind);) {
        u = g.ops[g.t[u].producer].in[0];
        if (g.t[u].kind != TS_ACT) break;
        chain.push_back(u);
      }
      for (size_t q = 0; q < chain.size(); ++q)
        for (int c : g.t[chain[q]].consumers)
          if (ew(g.ops[c].kind) && g.ops[c].in[0] == chain[q] &&
              std::find(chain.begin(), chain.end(), g.ops[c].out[0]) == chain.end())
            chain.push_back(g.ops[c].out[0]);
      for (int p = 2; p <= 16; p *= 2) {
        if (x.shape[1] % p || (x.shape[1] / p) % 8) break;
        for (int opt : {TS_RESIDE, TS_SWAP, TS_RECOMPUTE}) {
          Cand2 c;
          c.birth = birth[t];
          c.tensor = t;
          for (int u : chain) c.ch.push_back({u, u == t ? opt : ps.cfg[u].opt, p, ps.cfg[u].lead, 1});
          step2.push_back(opt == TS_RECOMPUTE ? with_feeders(c, t) : c);
        }
      }
    }
    // D-ATTR: band (height) splits of the bottleneck op's 4-D activations, with every tensor
    // a band-local op (ReLU, add, batch norm) ties to them — also only once the sample dim is
    // exhausted (Fig. 6: the attribute dim is what is left at batch 1); illegal groups (one
    // that feeds a flatten, a band without input rows) are dropped by attr_ok in consider()
    auto band_group = [&](int t) {
      std::vector<int> grp{t};
      auto local = [](int kind) { return kind == TS_OP_RELU || kind == TS_OP_ADD || kind == TS_OP_BATCHNORM; };
      for (size_t q = 0; q < grp.size(); ++q) {
        const Tensor& u = g.t[grp[q]];
        std::vector<int> nb;
        if (u.producer >= 0 && local(g.ops[u.producer].kind))
          for (int v : g.ops[u.producer].in) if (g.t[v].kind == TS_ACT) nb.push_back(v);
        for (int c : u.consumers)
          if (local(g.ops[c].kind)) nb.push_back(g.ops[c].out[0]);
        for (int v : nb)
          if (std::find(grp.begin(), grp.end(), v) == grp.end()) grp.push_back(v);
      }
      return grp;
    };
    std::vector<int> band_all;
    for (int t : split_cands) {
      const Tensor& x = g.t[t];
      if (no_split || x.ndim != 4) continue;
      const bool banded = is_attr(g, ps.cfg, t);  // a band split may grow finer
      bool sample_room = false;
      for (int p = 2 * ps.cfg[t].p; p <= 16 && !banded; p *= 2) sample_room |= g.samples % p == 0;
      if (sample_room) continue;
      const std::vector<int> grp = band_group(t);
      for (int u : grp)
        if (std::find(band_all.begin(), band_all.end(), u) == band_all.end()) band_all.push_back(u);
      for (int p = 2; p <= 16; p *= 2) {
        if (x.shape[1] % p) break;
        if (banded && p <= ps.cfg[t].p) continue;
        for (int opt : {TS_RESIDE, TS_SWAP, TS_RECOMPUTE}) {
          if (opt != TS_RESIDE && first_bw[t] < 0) continue;
          Cand2 c;
          c.birth = birth[t];
          c.tensor = t;
          for (int u : grp) c.ch.push_back({u, u == t ? opt : ps.cfg[u].opt, p, ps.cfg[u].lead, 2});
          step2.push_back(opt == TS_RECOMPUTE ? with_feeders(c, t) : c);
        }
      }
    }
    // the whole window micro-op in bands: its input's and its output's groups at once
    for (int p = 2; p <= 16 && band_all.size() > 1; p *= 2) {
      Cand2 c;
      for (int u : band_all)
        if (g.t[u].shape[1] % p == 0 && !(is_attr(g, ps.cfg, u) && ps.cfg[u].p >= p))
          c.ch.push_back({u, ps.cfg[u].opt, p, ps.cfg[u].lead, 2});
      if (c.ch.size() < 2) continue;
      c.birth = birth[c.ch[0].t];
      c.tensor = c.ch[0].t;
      step2.push_back(c);
    }
    // D-R8e: a recomputed tensor regenerated for the bottleneck (a replay chain member,
    // P:L294) is allocated piece by piece at its own split; splitting it finer shrinks
    // the replay's working set, so live recompute-opt tensors get split-only proposals.
    for (int t : live) {
      const Tensor& x = g.t[t];
      if (x.kind != TS_ACT || x.is_loss || own.count(t) || ps.cfg[t].opt != TS_RECOMPUTE) continue;
      const bool banded = is_attr(g, ps.cfg, t);
      for (int p = ps.cfg[t].p * 2; p <= 16 && !no_split && !banded; p *= 2) {
        if (g.samples % p) break;
        Cand2 c;
        c.birth = birth[t];
        c.tensor = t;
        c.ch = {{t, TS_RECOMPUTE, p, ps.cfg[t].lead}};
        step2.push_back(c);
      }
      // D-ATTR: with the sample dim exhausted, finer height bands for the tensor's group
      if (no_split || x.ndim != 4 || (!banded && g.samples % (2 * ps.cfg[t].p) == 0)) continue;
      const std::vector<int> grp = band_group(t);
      for (int p = banded ? ps.cfg[t].p * 2 : 2; p <= 16; p *= 2) {
        if (x.shape[1] % p) break;
        Cand2 c;
        c.birth = birth[t];
        c.tensor = t;
        for (int u : grp) c.ch.push_back({u, u == t ? TS_RECOMPUTE : ps.cfg[u].opt, p, ps.cfg[u].lead, 2});
        step2.push_back(c);
      }
    }
    // D-R8d: the whole micro-op split — every activation of the bottleneck op to the same
    // p at once.  Under op-major execution (R10) an input piece is released while the
    // output is produced only when both sides are split, so single-tensor splits can
    // show no gain (dM = 0) where the joint one does (e.g. VGG conv1 -> relu1).
    for (int p = 2; p <= 16 && !no_split; p *= 2) {
      if (g.samples % p) continue;
      Cand2 c;
      for (int t : split_cands)
        if (ps.cfg[t].p < p) c.ch.push_back({t, ps.cfg[t].opt, p, ps.cfg[t].lead});
      if (c.ch.size() < 2) continue;
      c.birth = birth[c.ch[0].t];
      c.tensor = c.ch[0].t;
      step2.push_back(c);
    }
    // step 3: score every proposal by re-simulation — dM = drop of the pool top over
    // the bottleneck op's items, dT = change of the predicted step time (timeline with
    // the profile, PCIe occupancy and swap-in stalls) — and take the best.
    // the bottleneck op's items: its micro-ops of this phase and, in the backward, the
    // recompute replays of its groups (they allocate for it)
    auto top_of_op = [&](const PlanState& st) {
      std::unordered_map<int, int> group_op;
      if (bwd_phase)
        for (const Item& it : st.ex.items)
          if (it.kind == IT_B) group_op[it.group] = it.op;
      uint64_t m = 0;
      for (size_t i = 0; i < st.ex.items.size(); ++i) {
        const Item& it = st.ex.items[i];
        if (it.kind == IT_SO || it.kind == IT_SI) continue;
        bool same_phase = ((int)i >= st.ex.fwd_end) == bwd_phase;
        if (!same_phase) continue;
        int op = it.op;
        if (it.kind == IT_R) {
          auto f = group_op.find(it.group);
          op = f == group_op.end() ? -1 : f->second;
        }
        if (op == bop) m = std::max(m, st.sim.top[i]);
      }
      return m;
    };
    const uint64_t cur_top = top_of_op(ps);
    const Cand2* best = nullptr;
    double best_ratio = 0, best_dm = 0;
    auto consider = [&](const Cand2& c) {
      PlanState cs;
      cs.cfg = ps.cfg;
      for (auto& chg : c.ch) {
        cs.cfg[chg.t].opt = chg.opt;
        cs.cfg[chg.t].p = chg.p;
        cs.cfg[chg.t].lead = chg.lead;
        cs.cfg[chg.t].lag = chg.opt == TS_SWAP ? chg.lag : 0;
        if (chg.dim >= 0) cs.cfg[chg.t].dim = chg.dim;
        if (chg.p == 1) cs.cfg[chg.t].dim = 0;
      }
      std::string why;
      if (!channel_ok(g, cs.cfg, why) || !attr_ok(g, cs.cfg, why)) return;
      plan_refresh(g, cs, &pr);
      uint64_t nt = top_of_op(cs);
      if (nt >= cur_top) return;
      double dm = double(cur_top - nt);
      double ratio = std::max(0.0, cs.predicted_s - ps.predicted_s) / dm;
      bool take = !best || ratio < best_ratio - 1e-18 ||
                  (std::fabs(ratio - best_ratio) <= 1e-18 &&
                   (dm > best_dm || (dm == best_dm && (c.birth < best->birth ||
                                                      (c.birth == best->birth && c.tensor < best->tensor)))));
      if (take) {
        best = &c;
        best_ratio = ratio;
        best_dm = dm;
      }
    };
    static const bool log = std::getenv("TS_PLAN_LOG") != nullptr;
    for (auto& c : step1) {
      consider(c);
      if (log) {
        PlanState cs;
        cs.cfg = ps.cfg;
        for (auto& chg : c.ch) {
          cs.cfg[chg.t].opt = chg.opt;
          cs.cfg[chg.t].p = chg.p;
          cs.cfg[chg.t].lead = chg.lead;
          cs.cfg[chg.t].lag = chg.opt == TS_SWAP ? chg.lag : 0;
        }
        plan_refresh(g, cs, &pr);
        std::fprintf(stderr, "  cand t=%d opt=%d lead=%d analytic=%.3g dT=%.3gms top %llu->%llu\n", c.tensor,
                     c.ch[0].opt, c.ch[0].lead, c.analytic, 1e3 * (cs.predicted_s - ps.predicted_s),
                     (unsigned long long)cur_top, (unsigned long long)top_of_op(cs));
      }
    }
    for (auto& c : step2) {
      consider(c);
      if (log && !best) {
        PlanState cs;
        cs.cfg = ps.cfg;
        for (auto& chg : c.ch) {
          cs.cfg[chg.t].opt = chg.opt;
          cs.cfg[chg.t].p = chg.p;
          cs.cfg[chg.t].lead = chg.lead;
          cs.cfg[chg.t].lag = chg.opt == TS_SWAP ? chg.lag : 0;
        }
        plan_refresh(g, cs, &pr);
        std::fprintf(stderr, "  cand2 t=%d n=%zu opt=%d p=%d top %llu->%llu\n", c.tensor, c.ch.size(), c.ch[0].opt,
                     c.ch[0].p, (unsigned long long)cur_top, (unsigned long long)top_of_op(cs));
      }
    }
    if (log && best)
      std::fprintf(stderr, "iter %d bottleneck item %d op %d (%s) top %.3f GB: pick t=%d opt=%d p=%d lead=%d ratio %.3g pred %.2f ms\n",
                   iter, bi, bop, bwd_phase ? "bwd" : "fwd", cur_top / 1e9, best->tensor, best->ch[0].opt,
                   best->ch[0].p, best->ch[0].lead, best_ratio, 1e3 * ps.predicted_s);
    if (!best && log) {
      std::fprintf(stderr, "stuck at item %d op %d (%s): live tensors\n", bi, bop, bwd_phase ? "bwd" : "fwd");
      for (int t = 0; t < n; ++t)
        if (ps.cfg[t].opt != TS_RESIDE || ps.cfg[t].p != 1)
          std::fprintf(stderr, "  cfg t=%d opt=%d p=%d\n", t, ps.cfg[t].opt, ps.cfg[t].p);
      for (int t : live)
        std::fprintf(stderr, "  t=%d opt=%d p=%d bytes=%llu own=%d first_bw=%d last_fw=%d\n", t, ps.cfg[t].opt,
                     ps.cfg[t].p, (unsigned long long)g.t[t].bytes, (int)own.count(t), first_bw[t], last_fw[t]);
      for (auto& e : ps.sim.trace)
        if (e.item == bi && e.kind == 0)
          std::fprintf(stderr, "  alloc@bi key=%d piece=%d bytes=%llu off=%llu\n", e.key, e.piece,
                       (unsigned long long)e.bytes, (unsigned long long)e.offset);
    }
    if (!best) {
      set_error("infeasible: no candidate left at op " + std::to_string(bop) + " (item " + std::to_string(bi) +
                ", needs " + std::to_string(ps.sim.top[bi]) + " B > budget " + std::to_string(budget) + ")");
      return TS_ERR_INFEASIBLE;
    }
    for (auto& chg : best->ch) {
      ps.cfg[chg.t].opt = chg.opt;
      ps.cfg[chg.t].p = chg.p;
      ps.cfg[chg.t].lead = chg.lead;
      ps.cfg[chg.t].lag = chg.opt == TS_SWAP ? chg.lag : 0;
      if (chg.dim >= 0) ps.cfg[chg.t].dim = chg.dim;
      if (chg.p == 1) ps.cfg[chg.t].dim = 0;
    }
  }
  set_error("planner did not converge");
  return TS_ERR_INFEASIBLE;
}

ts_status plan_greedy_lag(const Graph& g, uint64_t budget, const Profile& pr, PlanState& ps, uint32_t flags) {
  ts_status st = plan_greedy(g, budget, pr, ps, flags);
  if (st != TS_ERR_INFEASIBLE) return st;
  const std::string msg = ts_last_error();
  PlanState alt;
  if (plan_greedy(g, budget, pr, alt, flags | kPlanNoLag) == TS_OK) {
    ps = std::move(alt);
    return TS_OK;
  }
  set_error(msg);
  return st;
}

}  // namespace ts
