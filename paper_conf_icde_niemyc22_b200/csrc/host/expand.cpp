// Augmented-schedule expansion and pool simulation.
//   P:L262-264 Fig. 10 — split ops into p_num micro-ops, insert memory-option ops
//   P:L287             — in-place re-split (a micro-op reads a sub-range of a piece),
//                        best-fit allocation over one pre-allocated pool
//   P:L281             — swap-out begins at generation, swap-in at the previous op
//   P:L291             — compute / D2H / H2D streams, pre-allocated pool
//   P:L293-294 Fig. 11 — memory-centric recompute (regenerate for every backward use);
//                        with cache_bytes > 0 the LRU-based hybrid (reading D-LRU): regenerated
//                        pieces stay resident for later groups, least recently used ones are
//                        abandoned at the end of a group beyond cache_bytes
//   P:L56, P:L134      — allocate at the beginning, free at the end of an operation
#include <algorithm>
#include <functional>
#include <map>
#include <set>

#include "core.h"

namespace ts {

int piece_count(const Graph& g, const std::vector<Cfg>& cfg, int key) {
  int t = key >= g.n() ? key - g.n() : key;
  const Tensor& x = g.t[t];
  if (!x.sample || x.kind != TS_ACT) return 1;
  return cfg[t].p;
}

uint64_t piece_bytes(const Graph& g, const std::vector<Cfg>& cfg, int key) {
  int t = key >= g.n() ? key - g.n() : key;
  return g.t[t].bytes / uint64_t(piece_count(g, cfg, key));
}

// Channel (parameter-dim) split, reading D-CH (Fig. 6; oracle/sim.py
// check_channel): a 2-D activation split along its columns into p contiguous blocks.
bool is_chan(const Graph& g, const std::vector<Cfg>& cfg, int key) {
  int t = key >= g.n() ? key - g.n() : key;
  const Tensor& x = g.t[t];
  return x.sample && x.kind == TS_ACT && cfg[t].dim == 1 && cfg[t].p > 1;
}
bool channel_mode(const Graph& g, const std::vector<Cfg>& cfg, int op) {
  for (int x : g.ops[op].out)
    if (is_chan(g, cfg, x)) return true;
  return false;
}
static bool chan_ew(int kind) { return kind == TS_OP_RELU || kind == TS_OP_GELU || kind == TS_OP_TANH; }
// ops that map channel block k of their inputs to block k of their output: the elementwise
// ones, and for NHWC images (D-CH 4-D part) ReLU, add, batch norm and max pooling
bool chan_local(const Graph& g, int op) {
  const Op& o = g.ops[op];
  if (chan_ew(o.kind)) return true;
  return g.t[o.out[0]].ndim == 4 &&
         (o.kind == TS_OP_ADD || o.kind == TS_OP_BATCHNORM || o.kind == TS_OP_MAXPOOL);
}

bool channel_ok(const Graph& g, const std::vector<Cfg>& cfg, std::string& why) {
  for (int t = 0; t < g.n(); ++t) {
    if (cfg[t].dim < 0 || cfg[t].dim > 3)
      return (why = "split dim must be 0 (samples), 1 (channels), 2 (height) or 3 (width)"), false;
    if (!is_chan(g, cfg, t)) continue;
    const Tensor& x = g.t[t];
    const int p = cfg[t].p;
    if ((x.ndim != 2 && x.ndim != 4) || x.shape[x.ndim - 1] % p)
      return (why = "channel split needs a 2-D or NHWC activation with C % p == 0"), false;
    const Op& po = g.ops[x.producer];
    const int xi = po.in.empty() ? -1 : po.in[0];
    if (po.kind == TS_OP_LINEAR || (po.kind == TS_OP_CONV2D && x.ndim == 4)) {
      if (!is_chan(g, cfg, xi) && g.t[xi].kind == TS_ACT && cfg[xi].p != 1)
        return (why = "a channel-split linear output needs an unsplit or channel-split input"), false;
      if (po.kind == TS_OP_CONV2D && is_chan(g, cfg, xi))
        return (why = "a channel-split conv output needs an unsplit input"), false;
    } else if (chan_local(g, po.id)) {
      for (int u : po.in)
        if (g.t[u].kind == TS_ACT && (!is_chan(g, cfg, u) || cfg[u].p != p))
          return (why = "an elementwise producer needs a channel-split input of the same p"), false;
    } else {
      return (why = "only linear / conv / relu / gelu / tanh / add / batchnorm / maxpool can write channel blocks"), false;
    }
    for (int c : x.consumers) {
      const Op& co = g.ops[c];
      const int y = co.out[0];
      if (co.kind == TS_OP_LINEAR && co.in[0] == t && x.ndim == 2) {
        if (!is_chan(g, cfg, y) && g.t[y].kind == TS_ACT && cfg[y].p != 1)
          return (why = "a linear reading channel blocks needs an unsplit or channel-split output"), false;
      } else if (co.kind == TS_OP_CONV2D && x.ndim == 4) {
        if (cfg[y].dim != 0 && cfg[y].p > 1)
          return (why = "a conv reading channel blocks needs an unsplit or sample-split output"), false;
      } else if (chan_local(g, c)) {
        if (!is_chan(g, cfg, y) || cfg[y].p != p)
          return (why = "an elementwise consumer needs a channel-split output of the same p"), false;
      } else {
        return (why = "only linear (as X) / conv / elementwise ops can read channel blocks"), false;
      }
    }
  }
  return true;
}

// Attribute split, reading D-ATTR (Fig. 10; oracle/sim.py check_attr): a
// 4-D NHWC activation split along H (dim 2) into p bands [B, H/p, W, C] or along W (dim 3)
// into [B, H, W/p, C].
bool is_attr(const Graph& g, const std::vector<Cfg>& cfg, int key) {
  int t = key >= g.n() ? key - g.n() : key;
  const Tensor& x = g.t[t];
  return x.sample && x.kind == TS_ACT && (cfg[t].dim == 2 || cfg[t].dim == 3) && cfg[t].p > 1;
}
bool attr_mode(const Graph& g, const std::vector<Cfg>& cfg, int op) {
  for (int x : g.ops[op].out)
    if (is_attr(g, cfg, x)) return true;
  return false;
}
static bool attr_local(int kind) { return kind == TS_OP_RELU || kind == TS_OP_ADD || kind == TS_OP_BATCHNORM; }
bool attr_window(int kind) { return kind == TS_OP_CONV2D || kind == TS_OP_MAXPOOL; }
bool attr_staged(const Graph& g, const std::vector<Cfg>& cfg, int op) {
  const Op& o = g.ops[op];
  return attr_window(o.kind) && (is_attr(g, cfg, o.in[0]) || attr_mode(g, cfg, op) ||
                                 (o.kind == TS_OP_CONV2D && is_chan(g, cfg, o.in[0])));  // D-CH staged merge
}

Window window_geom(const Graph& g, int op, int axis) {
  const Op& o = g.ops[op];
  if (o.kind == TS_OP_CONV2D) return {int(g.t[o.in[1]].shape[axis]), int(o.ia[0]), int(o.ia[1])};
  return {int(o.ia[0]), int(o.ia[1]), int(o.ia[2])};
}

Staged staged_rect(const Graph& g, const std::vector<Cfg>& cfg, int op, int k, int P) {
  const Op& o = g.ops[op];
  const int y = o.out[0];
  const bool band = is_attr(g, cfg, y);
  int64_t lo[3] = {0, 0, 0}, cnt[3] = {0, 0, 0};
  for (int axis = 1; axis <= 2; ++axis) {
    const Window w = window_geom(g, op, axis);
    const bool here = band && attr_axis(cfg, y) == axis;  // the output's band axis
    const int64_t ho = g.t[y].shape[axis];
    const int64_t hb = here ? ho / P : ho;
    const int64_t kk = here ? k : 0;
    lo[axis] = kk * hb * w.stride - w.pad;
    cnt[axis] = ((kk + 1) * hb - 1) * w.stride - w.pad + w.R - 1 - lo[axis] + 1;
  }
  return {lo[1], cnt[1], lo[2], cnt[2], band ? g.samples : g.samples / P};
}

uint64_t staged_bytes(const Graph& g, const std::vector<Cfg>& cfg, int op, int k, int P) {
  const Tensor& x = g.t[g.ops[op].in[0]];
  const Staged s = staged_rect(g, cfg, op, k, P);
  return uint64_t(s.nb * s.hs * s.ws * x.shape[3]) * uint64_t(dtype_bytes(x.dtype));
}

bool attr_ok(const Graph& g, const std::vector<Cfg>& cfg, std::string& why) {
  for (int t = 0; t < g.n(); ++t) {
    if (!is_attr(g, cfg, t)) continue;
    const Tensor& x = g.t[t];
    const int p = cfg[t].p, d = cfg[t].dim;
    if (x.ndim != 4 || x.shape[attr_axis(cfg, t)] % p)
      return (why = "a band split needs an NHWC activation whose H (W) p divides"), false;
    auto same = [&](int u) { return is_attr(g, cfg, u) && cfg[u].p == p && cfg[u].dim == d; };
    const Op& po = g.ops[x.producer];
    if (attr_local(po.kind)) {
      for (int u : po.in)
        if (g.t[u].kind == TS_ACT && !same(u))
          return (why = "a band-local producer needs band-split inputs of the same p and dim"), false;
    } else if (attr_window(po.kind)) {
      const int u = po.in[0];
      if (!is_attr(g, cfg, u) && cfg[u].p != 1)
        return (why = "a band-split window output needs an unsplit or band-split input"), false;
    } else {
      return (why = "only conv2d / maxpool / relu / add / batchnorm can write bands"), false;
    }
    for (int c : x.consumers) {
      const Op& co = g.ops[c];
      const int y = co.out[0];
      if (attr_local(co.kind)) {
        if (!same(y)) return (why = "a band-local consumer needs a band-split output of the same p and dim"), false;
      } else if (attr_window(co.kind)) {
        if (is_chan(g, cfg, y)) return (why = "a window op reading bands cannot write channel blocks"), false;
      } else {
        return (why = "only conv2d / maxpool / relu / add / batchnorm can read bands"), false;
      }
    }
  }
  // every band of a band-mode window op reads at least one input row
  for (auto& o : g.ops) {
    if (!attr_window(o.kind) || !attr_mode(g, cfg, o.id)) continue;
    const int P = cfg[o.out[0]].p;
    const int ax = attr_axis(cfg, o.out[0]);
    const int64_t H = g.t[o.in[0]].shape[ax];
    for (int k = 0; k < P; ++k) {
      const Staged s = staged_rect(g, cfg, o.id, k, P);
      const int64_t lo = ax == 1 ? s.rlo : s.clo, cnt = ax == 1 ? s.hs : s.ws;
      if (std::max<int64_t>(lo, 0) > std::min<int64_t>(lo + cnt - 1, H - 1))
        return (why = "a band of a window op reads no input row"), false;
    }
  }
  return true;
}

uint64_t Expansion::bytes(const Graph& g, const std::vector<Cfg>& cfg, PieceKey pc) const {
  if (pk_key(pc) >= 2 * g.n()) return temp_bytes.at(pc);
  return piece_bytes(g, cfg, pk_key(pc));
}

void expand(const Graph& g, const std::vector<Cfg>& cfg, Expansion& ex, uint64_t cache_bytes) {
  const int n = g.n();
  ex = Expansion();
  ex.P.assign(g.ops.size(), 1);
  std::vector<char> cm(g.ops.size(), 0), am(g.ops.size(), 0), st(g.ops.size(), 0);
  for (auto& o : g.ops) {
    int P = 1;
    cm[o.id] = channel_mode(g, cfg, o.id) ? 1 : 0;
    am[o.id] = attr_mode(g, cfg, o.id) ? 1 : 0;
    st[o.id] = attr_staged(g, cfg, o.id) ? 1 : 0;
    if (cm[o.id]) {  // D-CH: one micro-op per channel block of the output
      for (int x : o.out)
        if (is_chan(g, cfg, x)) P = std::max(P, piece_count(g, cfg, x));
    } else if (am[o.id]) {  // D-ATTR: one micro-op per band of the output
      for (int x : o.out)
        if (is_attr(g, cfg, x)) P = std::max(P, piece_count(g, cfg, x));
    } else {
      for (int x : o.in)
        if (g.t[x].sample && !is_chan(g, cfg, x) && !is_attr(g, cfg, x)) P = std::max(P, piece_count(g, cfg, x));
      for (int x : o.out)
        if (g.t[x].sample && !is_chan(g, cfg, x) && !is_attr(g, cfg, x)) P = std::max(P, piece_count(g, cfg, x));
    }
    ex.P[o.id] = P;
  }
  // the pieces of t (or of its gradient) micro-op k of op `op` touches (D-CH: a channel-split
  // tensor is block k in its channel-mode producer / elementwise consumer, else all blocks;
  // D-ATTR: a band-split window input is the bands holding the staged rows, else band k)
  auto pieces = [&](int t, int k, int P, int op) -> std::vector<int> {
    if (!g.t[t].sample) return {0};
    if (is_chan(g, cfg, t)) {
      const Op& o = g.ops[op];
      if (cm[op] && (std::find(o.out.begin(), o.out.end(), t) != o.out.end() || chan_local(g, op))) return {k};
      std::vector<int> all(piece_count(g, cfg, t));
      for (size_t j = 0; j < all.size(); ++j) all[j] = int(j);
      return all;
    }
    if (is_attr(g, cfg, t)) {
      const Op& o = g.ops[op];
      if (attr_window(o.kind) && o.in[0] == t) {
        const Staged s = staged_rect(g, cfg, op, k, P);
        const int ax = attr_axis(cfg, t);
        const int64_t H = g.t[t].shape[ax], hb = H / piece_count(g, cfg, t);
        const int64_t lo0 = ax == 1 ? s.rlo : s.clo, cnt = ax == 1 ? s.hs : s.ws;
        const int64_t lo = std::max<int64_t>(lo0, 0), hi = std::min<int64_t>(lo0 + cnt - 1, H - 1);
        std::vector<int> js;
        for (int64_t j = lo / hb; j <= hi / hb; ++j) js.push_back(int(j));
        return js;
      }
      return {k};
    }
    return {k * piece_count(g, cfg, t) / P};
  };
  auto add_temps = [&](Item& it, int op, int k, int P, bool bwd) {
    if (!st[op]) return;
    const uint64_t b = staged_bytes(g, cfg, op, k, P);
    it.temps.push_back(pk(2 * n + op, k));
    const Tensor& x = g.t[g.ops[op].in[0]];
    if (bwd && x.kind == TS_ACT && x.needs_grad) it.temps.push_back(pk(3 * n + op, k));  // (the image: no dX)
    for (PieceKey pc : it.temps) ex.temp_bytes[pc] = b;
  };
  std::vector<Item>& items = ex.items;
  // ---- forward phase: op-major micro-ops (R10) ------------------------------
  for (int o : g.order) {
    const Op& op = g.ops[o];
    int P = ex.P[o];
    for (int k = 0; k < P; ++k) {
      Item it;
      it.kind = IT_F;
      it.op = o;
      it.k = k;
      for (int x : op.in)
        if (g.t[x].sample)
          for (int j : pieces(x, k, P, o)) it.reads.push_back(pk(x, j));
      if (batch_reduce(op.kind) && k == 0 && !cm[o])  // full-batch statistics (R13; channel mode: per block)
        for (int x : op.in)
          if (g.t[x].sample)
            for (int j = 0; j < piece_count(g, cfg, x); ++j)
              if (std::find(it.reads.begin(), it.reads.end(), pk(x, j)) == it.reads.end()) it.reads.push_back(pk(x, j));
      for (int x : op.out)
        for (int j : pieces(x, k, P, o)) it.writes.push_back(pk(x, j));
      add_temps(it, o, k, P, false);
      items.push_back(std::move(it));
    }
  }
  ex.fwd_end = (int)items.size();
  // ---- backward phase: reverse order, replays inline --------------------------
  // D-LRU cache: regenerated pieces still resident, least recently used first
  std::vector<std::pair<PieceKey, uint64_t>> cache;
  auto cache_find = [&](PieceKey pc) {
    for (size_t i = 0; i < cache.size(); ++i)
      if (cache[i].first == pc) return int(i);
    return -1;
  };
  int gid = 0;
  for (auto rit = g.order.rbegin(); rit != g.order.rend(); ++rit) {
    const Op& op = g.ops[*rit];
    if (!op.has_bwd) continue;
    int P = ex.P[op.id];
    for (int k = 0; k < P; ++k) {
      std::vector<Item> group;
      std::set<PieceKey> regenerated;
      std::function<void(int, int)> regen = [&](int t, int j) {
        const Tensor& x = g.t[t];
        if (x.kind != TS_ACT || cfg[t].opt != TS_RECOMPUTE) return;
        if (regenerated.count(pk(t, j))) return;
        int ci = cache_find(pk(t, j));
        if (ci >= 0) {  // D-LRU hit: resident since an earlier group; now most recently used
          auto e = cache[ci];
          cache.erase(cache.begin() + ci);
          cache.push_back(e);
          regenerated.insert(pk(t, j));
          return;
        }
        const Op& po = g.ops[x.producer];
        int Q = ex.P[po.id];
        int pt = piece_count(g, cfg, t);
        for (int kk = j * Q / pt; kk < (j + 1) * Q / pt; ++kk) {
          for (int u : po.in)
            if (g.t[u].sample)
              for (int jj : pieces(u, kk, Q, po.id)) regen(u, jj);
          Item r;
          r.kind = IT_R;
          r.op = po.id;
          r.k = kk;
          r.group = gid;
          for (int u : po.in)
            if (g.t[u].sample)
              for (int jj : pieces(u, kk, Q, po.id)) r.reads.push_back(pk(u, jj));
          r.writes.push_back(pk(t, j));
          add_temps(r, po.id, kk, Q, false);
          group.push_back(std::move(r));
        }
        regenerated.insert(pk(t, j));
        cache.push_back({pk(t, j), piece_bytes(g, cfg, t)});
      };
      std::vector<PieceKey> saved;
      for (int t : op.saved)
        for (int j : pieces(t, k, P, op.id)) saved.push_back(pk(t, j));
      if (batch_reduce(op.kind) && k == 0 && !cm[op.id])
        for (int t : op.saved)
          for (int j = 0; j < piece_count(g, cfg, t); ++j)
            if (std::find(saved.begin(), saved.end(), pk(t, j)) == saved.end()) saved.push_back(pk(t, j));
      for (PieceKey s : saved) regen(pk_key(s), pk_j(s));
      Item b;
      b.kind = IT_B;
      b.op = op.id;
      b.k = k;
      b.group = gid;
      add_temps(b, op.id, k, P, true);
      b.reads = saved;
      for (int x : op.out)
        if (!g.t[x].is_loss && g.t[x].needs_grad) {
          for (int j : pieces(x, k, P, op.id)) b.reads.push_back(pk(n + x, j));
          if (batch_reduce(op.kind) && k == 0 && !cm[op.id])
            for (int j = 0; j < piece_count(g, cfg, x); ++j)
              if (std::find(b.reads.begin(), b.reads.end(), pk(n + x, j)) == b.reads.end())
                b.reads.push_back(pk(n + x, j));
        }
      for (int x : op.in)
        if (g.t[x].kind == TS_ACT && g.t[x].needs_grad) {
          for (int j : pieces(x, k, P, op.id)) {
            PieceKey w = pk(n + x, j);
            if (std::find(b.writes.begin(), b.writes.end(), w) == b.writes.end()) b.writes.push_back(w);
          }
        }
      group.push_back(std::move(b));
      for (auto& it : group) items.push_back(std::move(it));
      ++gid;
      // abandon the least recently used regenerated pieces beyond the cache limit
      uint64_t used = 0;
      for (auto& e : cache) used += e.second;
      while (!cache.empty() && used > cache_bytes) {
        used -= cache.front().second;
        cache.erase(cache.begin());
      }
    }
  }
  const int nitems = (int)items.size();
  // ---- lifetimes (R3, R12) --------------------------------------------------
  std::map<PieceKey, std::vector<int>> touches;
  for (int i = 0; i < nitems; ++i) {
    for (PieceKey p : items[i].writes) touches[p].push_back(i);
    for (PieceKey p : items[i].reads) touches[p].push_back(i);
  }
  std::vector<std::vector<PieceKey>> alloc_at(nitems), free_after(nitems), so_after(nitems), si_before(nitems);
  std::vector<std::vector<PieceKey>> lag_free(nitems);  // D-LAG: swapped-out pieces freed after item i
  std::set<PieceKey> lagged;
  for (auto& [pc, idx] : touches) {
    std::sort(idx.begin(), idx.end());
    idx.erase(std::unique(idx.begin(), idx.end()), idx.end());
    int key = pk_key(pc);
    int first = idx.front(), lastt = idx.back();
    if (key >= n) {  // gradient piece
      alloc_at[first].push_back(pc);
      free_after[lastt].push_back(pc);
      continue;
    }
    const Tensor& x = g.t[key];
    if (x.kind == TS_INPUT || x.kind == TS_LABEL) {
      free_after[lastt].push_back(pc);
      continue;
    }
    if (x.is_loss) {
      alloc_at[first].push_back(pc);
      continue;
    }
    int last_fw = -1, first_bw = -1;
    for (int i : idx) {
      if (i < ex.fwd_end) last_fw = i;
      else if (first_bw < 0) first_bw = i;
    }
    alloc_at[first].push_back(pc);  // first touch is its producing forward micro-op
    int opt = cfg[key].opt;
    if (first_bw < 0 || opt == TS_RESIDE) {
      free_after[lastt].push_back(pc);
    } else if (opt == TS_SWAP) {
      so_after[last_fw].push_back(pc);
      int pos = std::max(first_bw - std::max(1, cfg[key].lead), ex.fwd_end);
      si_before[pos].push_back(pc);
      free_after[lastt].push_back(pc);
      // D-LAG: the swapped-out range returns to the pool after the lag-th compute item
      // behind the swap-out (the copy's time), always before the swap-in
      const int q = std::min(last_fw + cfg[key].lag, pos - 1);
      if (cfg[key].lag > 0 && q > last_fw) {
        lag_free[q].push_back(pc);
        lagged.insert(pc);
      }
    } else {  // recompute: forward lifetime, then one residency per regeneration
      free_after[last_fw].push_back(pc);
      // a residency starts at the group's first replay writing the piece and ends at its
      // last touch before the next regeneration (memory-centric: one per group)
      std::vector<int> starts;
      std::set<int> seen;
      for (int i : idx)
        if (i >= ex.fwd_end && items[i].kind == IT_R && !seen.count(items[i].group) &&
            std::find(items[i].writes.begin(), items[i].writes.end(), pc) != items[i].writes.end()) {
          seen.insert(items[i].group);
          starts.push_back(i);
        }
      for (size_t a = 0; a < starts.size(); ++a) {
        const int st = starts[a], end = a + 1 < starts.size() ? starts[a + 1] : nitems;
        int last = st;
        for (int i : idx)
          if (i >= st && i < end) last = std::max(last, i);
        alloc_at[st].push_back(pc);
        free_after[last].push_back(pc);
      }
    }
  }
  // ---- final list with swap-out / swap-in items ------------------------------
  std::vector<Item> fin;
  fin.reserve(nitems * 2);
  for (int i = 0; i < nitems; ++i) {
    std::sort(si_before[i].begin(), si_before[i].end());
    for (PieceKey pc : si_before[i]) {
      Item si;
      si.kind = IT_SI;
      si.writes.push_back(pc);
      ex.alloc_at.push_back({pc});
      ex.free_after.push_back({});
      fin.push_back(std::move(si));
    }
    const Item& it = items[i];
    std::vector<PieceKey> order;
    auto& al = alloc_at[i];
    for (PieceKey p : it.writes)
      if (std::find(al.begin(), al.end(), p) != al.end() && std::find(order.begin(), order.end(), p) == order.end())
        order.push_back(p);
    for (PieceKey p : it.reads)
      if (std::find(al.begin(), al.end(), p) != al.end() && std::find(order.begin(), order.end(), p) == order.end())
        order.push_back(p);
    order.insert(order.end(), it.temps.begin(), it.temps.end());  // staging temporaries last (D-ATTR)
    std::vector<PieceKey> fr = free_after[i];
    fr.insert(fr.end(), lag_free[i].begin(), lag_free[i].end());
    fr.insert(fr.end(), it.temps.begin(), it.temps.end());
    std::sort(fr.begin(), fr.end());
    ex.alloc_at.push_back(order);
    ex.free_after.push_back(fr);
    fin.push_back(it);
    std::sort(so_after[i].begin(), so_after[i].end());
    for (PieceKey pc : so_after[i]) {
      Item so;
      so.kind = IT_SO;
      so.reads.push_back(pc);
      ex.alloc_at.push_back({});
      ex.free_after.push_back(lagged.count(pc) ? std::vector<PieceKey>{} : std::vector<PieceKey>{pc});
      fin.push_back(std::move(so));
    }
  }
  // fwd_end in the final numbering = index of the first backward-phase item
  int fe = 0;
  for (size_t i = 0; i < fin.size(); ++i)
    if (fin[i].kind == IT_F || fin[i].kind == IT_SO) fe = (int)i + 1;
  ex.items = std::move(fin);
  ex.fwd_end = fe;
}

// ---- pool --------------------------------------------------------------------
void Pool::reset(uint64_t base, uint64_t capacity) {
  cap_ = capacity;
  extent_ = base;
  free_.clear();
  if (capacity > base) free_.push_back({base, capacity - base});
}

bool Pool::alloc(uint64_t bytes, uint64_t* off) {
  uint64_t need = align_up(bytes);
  int best = -1;
  for (int i = 0; i < (int)free_.size(); ++i) {
    if (free_[i].first + free_[i].second == cap_) continue;  // tail: last resort
    if (free_[i].second >= need && (best < 0 || free_[i].second < free_[best].second)) best = i;
  }
  if (best < 0) {
    if (free_.empty()) return false;
    int t = (int)free_.size() - 1;
    if (free_[t].first + free_[t].second != cap_ || free_[t].second < need) return false;
    best = t;
  }
  *off = free_[best].first;
  if (free_[best].second == need) free_.erase(free_.begin() + best);
  else {
    free_[best].first += need;
    free_[best].second -= need;
  }
  extent_ = std::max(extent_, *off + need);
  return true;
}

void Pool::release(uint64_t off, uint64_t bytes) {
  uint64_t need = align_up(bytes);
  size_t i = 0;
  while (i < free_.size() && free_[i].first < off) ++i;
  free_.insert(free_.begin() + i, {off, need});
  if (i + 1 < free_.size() && free_[i].first + free_[i].second == free_[i + 1].first) {
    free_[i].second += free_[i + 1].second;
    free_.erase(free_.begin() + i + 1);
  }
  if (i > 0 && free_[i - 1].first + free_[i - 1].second == free_[i].first) {
    free_[i - 1].second += free_[i].second;
    free_.erase(free_.begin() + i);
  }
}

uint64_t Pool::top() const {
  if (!free_.empty() && free_.back().first + free_.back().second == cap_) return free_.back().first;
  return cap_;
}

bool simulate(const Graph& g, const std::vector<Cfg>& cfg, const Expansion& ex, uint64_t capacity,
              SimResult& r, std::vector<std::vector<std::pair<PieceKey, uint64_t>>>* placements) {
  r = SimResult();
  Pool pool;
  pool.reset(g.static_bytes, capacity);
  std::unordered_map<PieceKey, uint64_t> where;
  uint64_t live = 0, peak = 0, top = g.static_bytes;
  struct Fence {
    uint64_t off, len;
    int so;
  };
  std::vector<Fence> pend_cs, pend_h2d;
  r.wait_so.assign(ex.items.size(), {});
  int cur_item = -1;
  int64_t seq = 0;
  bool ok = true;
  auto do_alloc = [&](int item, PieceKey pc) {
    uint64_t b = ex.bytes(g, cfg, pc), off = 0;
    if (!pool.alloc(b, &off)) {
      ok = false;
      return;
    }
    where[pc] = off;
    r.offset[pc] = off;
    live += align_up(b);
    if (item >= 0) {
      auto& pend = ex.items[item].kind == IT_SI ? pend_h2d : pend_cs;
      const uint64_t len = align_up(b);
      for (size_t f = 0; f < pend.size();) {
        if (off < pend[f].off + pend[f].len && pend[f].off < off + len) {
          r.wait_so[item].push_back(pend[f].so);
          pend.erase(pend.begin() + f);
        } else {
          ++f;
        }
      }
    }
    r.trace.push_back({seq++, item, 0, pk_key(pc), pk_j(pc), off, b});
    if (placements && item >= 0) (*placements)[item].push_back({pc, off});
  };
  auto do_free = [&](int item, PieceKey pc) {
    uint64_t b = ex.bytes(g, cfg, pc);
    auto it = where.find(pc);
    uint64_t off = it->second;
    where.erase(it);
    pool.release(off, b);
    live -= align_up(b);
    r.trace.push_back({seq++, item, 1, pk_key(pc), pk_j(pc), off, b});
  };
  if (placements) placements->assign(ex.items.size(), {});
  for (auto& t : g.t)
    if (t.kind == TS_INPUT || t.kind == TS_LABEL) do_alloc(-1, pk(t.id, 0));
  if (!ok) return false;
  peak = live;
  r.top.resize(ex.items.size());
  r.live.resize(ex.items.size());
  for (size_t i = 0; i < ex.items.size(); ++i) {
    const Item& it = ex.items[i];
    for (PieceKey pc : ex.alloc_at[i]) {
      do_alloc((int)i, pc);
      if (!ok) return false;
    }
    top = pool.top();
    r.top[i] = top;
    r.live[i] = live;
    peak = std::max(peak, live);
    if (it.kind == IT_SO) r.d2h += ex.bytes(g, cfg, it.reads[0]);
    else if (it.kind == IT_SI) r.h2d += ex.bytes(g, cfg, it.writes[0]);
    else if (it.kind == IT_R) ++r.n_replay;
    else ++r.n_compute;
    if (it.kind == IT_SO) {
      const PieceKey pc = it.reads[0];
      Fence f{where.at(pc), align_up(ex.bytes(g, cfg, pc)), (int)i};
      pend_cs.push_back(f);
      pend_h2d.push_back(f);
    }
    for (PieceKey pc : ex.free_after[i]) do_free((int)i, pc);
  }
  (void)cur_item;
  std::vector<PieceKey> rest;
  for (auto& kv : where) rest.push_back(kv.first);
  std::sort(rest.begin(), rest.end());
  for (PieceKey pc : rest) do_free((int)ex.items.size(), pc);
  r.peak_live = g.static_bytes + peak;
  r.peak_extent = pool.extent();
  return true;
}

}  // namespace ts
