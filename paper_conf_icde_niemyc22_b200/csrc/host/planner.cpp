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
  std::unordered_map<PieceKey, double> ready;
  double clock = 0, d2h_free = 0, h2d_free = 0;
  for (size_t i = 0; i < ni; ++i) {
    const Item& it = items[i];
    if (it.kind == IT_SO) {
      double s = std::max(clock, d2h_free);
      double e = s + double(piece_bytes(g, ps.cfg, pk_key(it.reads[0]))) / pr.hw.d2h_bw;
      busy_d2h.push_back({s, e});
      d2h_free = e;
      continue;
    }
    if (it.kind == IT_SI) {
      double s = std::max(clock, h2d_free);
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
    int l = lg2(ps.ex.P[it.op]);
    double t = (it.kind == IT_B ? pr.tb[it.op][l] : pr.tf[it.op][l]) / double(ps.ex.P[it.op]);
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
  expand(g, ps.cfg, ps.ex);
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

ts_status plan_greedy(const Graph& g, uint64_t budget, const Profile& pr, PlanState& ps) {
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
    plan_refresh(g, ps, nullptr);
    const auto& items = ps.ex.items;
    int bi = -1;
    for (size_t i = 0; i < items.size(); ++i)
      if (ps.sim.top[i] > budget) {
        bi = (int)i;
        break;
      }
    if (bi < 0) {
      plan_refresh(g, ps, &pr);
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
    Cand best;
    // ---- step 1: non-split options on live tensors that are neither inputs nor
    // outputs of the bottleneck op (Eq. 2, Eq. 3, R6) --------------------------
    for (int t : live) {
      const Tensor& x = g.t[t];
      if (x.kind != TS_ACT || x.is_loss || ps.cfg[t].opt != TS_RESIDE || own.count(t)) continue;
      if (first_bw[t] < 0) continue;  // not held for backward: nothing to gain
      if (!bwd_phase && last_fw[t] >= bi) continue;  // still read later in the forward pass
      if (bwd_phase && first_bw[t] - std::max(1, ps.cfg[t].lead) <= bi) {
        // a swap would already be back by i; a recompute would be live in this group
        continue;
      }
      double dm = double(x.bytes);
      Cand c1;
      c1.valid = true;
      c1.tensor = t;
      c1.birth = birth[t];
      c1.p = ps.cfg[t].p;
      c1.opt = TS_SWAP;
      c1.ratio = swap_cost(t, dm) / dm;
      if (better(c1, best)) best = c1;
      c1.opt = TS_RECOMPUTE;
      c1.ratio = double(bw_ops[t].size()) * rc_time(rc_time, t, 0) / dm;
      if (better(c1, best)) best = c1;
    }
    // ---- step 2: split options on the bottleneck op's own tensors (Eq. 6) -----
    auto top_of_op = [&](const PlanState& s) {
      uint64_t m = 0;
      for (size_t i = 0; i < s.ex.items.size(); ++i) {
        const Item& it = s.ex.items[i];
        if (it.kind == IT_SO || it.kind == IT_SI) continue;
        bool same_phase = ((int)i >= s.ex.fwd_end) == bwd_phase;
        if (same_phase && it.op == bop) m = std::max(m, s.sim.top[i]);
      }
      return m;
    };
    uint64_t cur_top = top_of_op(ps);
    std::vector<int> split_cands;
    for (int x : g.ops[bop].in)
      if (g.t[x].kind == TS_ACT && !g.t[x].is_loss) split_cands.push_back(x);
    for (int x : g.ops[bop].out)
      if (g.t[x].kind == TS_ACT && !g.t[x].is_loss) split_cands.push_back(x);
    for (int t : split_cands) {
      for (int p = 2; p <= 16; p *= 2) {
        if (p <= ps.cfg[t].p || g.samples % p) continue;
        for (int opt : {TS_RESIDE, TS_SWAP, TS_RECOMPUTE}) {
          if (opt != TS_RESIDE && first_bw[t] < 0) continue;
          PlanState cand;
          cand.cfg = ps.cfg;
          cand.cfg[t].opt = opt;
          cand.cfg[t].p = p;
          plan_refresh(g, cand, nullptr);
          uint64_t nt = top_of_op(cand);
          if (nt >= cur_top) continue;
          double dm = double(cur_top - nt);
          double micro = 0;
          if (opt == TS_SWAP) micro = swap_cost(t, double(g.t[t].bytes) / p);
          if (opt == TS_RECOMPUTE) micro = double(bw_ops[t].size()) * rc_time(rc_time, t, 0) / p;
          double dsplit = 0;
          std::set<int> ops_t(g.t[t].consumers.begin(), g.t[t].consumers.end());
          ops_t.insert(g.t[t].producer);
          for (int o : ops_t) {
            int l0 = lg2(ps.ex.P[o]), l1 = lg2(cand.ex.P[o]);
            dsplit += pr.tf[o][l1] - pr.tf[o][l0];
            if (g.ops[o].has_bwd) dsplit += pr.tb[o][l1] - pr.tb[o][l0];
          }
          Cand c2;
          c2.valid = true;
          c2.tensor = t;
          c2.birth = birth[t];
          c2.opt = opt;
          c2.p = p;
          c2.ratio = (double(p - 1) * micro + std::max(0.0, dsplit)) / dm;
          if (better(c2, best)) best = c2;
        }
      }
    }
    if (!best.valid) {
      set_error("infeasible: no candidate left at op " + std::to_string(bop) + " (item " +
                std::to_string(bi) + ", needs " + std::to_string(ps.sim.top[bi]) + " B > budget " +
                std::to_string(budget) + ")");
      return TS_ERR_INFEASIBLE;
    }
    ps.cfg[best.tensor].opt = best.opt;
    ps.cfg[best.tensor].p = best.p;
  }
  set_error("planner did not converge");
  return TS_ERR_INFEASIBLE;
}

}  // namespace ts
