// Graph definition, validation, analysis and the Alg. 1 execution schedule.
//   P:L56 §II   — DFG: ops are nodes, tensors are edges
//   P:L62-83    — Alg. 1 "Construct Execution Schedule", DFS-manner topo sort;
//                 line 5 read as ref_cnt -= 1 and line 6 as == 0
#include <algorithm>
#include <cstring>
#include <functional>
#include <sstream>

#include "core.h"

namespace ts {

namespace {

bool fail(const std::string& m) {
  set_error(m);
  return false;
}

int64_t last(const Tensor& t) { return t.shape[t.ndim - 1]; }

bool same_shape(const Tensor& a, const Tensor& b) {
  if (a.ndim != b.ndim) return false;
  for (int i = 0; i < a.ndim; ++i)
    if (a.shape[i] != b.shape[i]) return false;
  return true;
}

// Shape/dtype validation per op kind.
bool validate_op(const Graph& g, const Op& o, std::string& why) {
  auto T = [&](int i) -> const Tensor& { return g.t[i]; };
  auto need = [&](size_t ni, size_t no) {
    if (o.in.size() != ni || o.out.size() != no) {
      why = "wrong number of inputs/outputs";
      return false;
    }
    return true;
  };
  switch (o.kind) {
    case TS_OP_LINEAR: {
      if (!need(3, 1)) return false;
      const Tensor &x = T(o.in[0]), &w = T(o.in[1]), &b = T(o.in[2]), &y = T(o.out[0]);
      if (x.ndim != 2 || w.ndim != 2 || b.ndim != 1 || y.ndim != 2) return (why = "linear ranks"), false;
      if (x.shape[1] != w.shape[1] || b.shape[0] != w.shape[0] || y.shape[0] != x.shape[0] ||
          y.shape[1] != w.shape[0])
        return (why = "linear shapes"), false;
      if (w.kind != TS_PARAM || b.kind != TS_PARAM) return (why = "linear W/b must be params"), false;
      return true;
    }
    case TS_OP_RELU: case TS_OP_GELU: case TS_OP_TANH: case TS_OP_SOFTMAX: case TS_OP_DROPOUT:
      if (!need(1, 1)) return false;
      if (!same_shape(T(o.in[0]), T(o.out[0]))) return (why = "elementwise shapes"), false;
      if (o.kind == TS_OP_DROPOUT && (o.fa.size() < 1 || o.ia.size() < 1)) return (why = "dropout attrs"), false;
      if (o.kind == TS_OP_SOFTMAX && !o.ia.empty() && o.ia[0] != 0) {  // causal: square [.., s, s] scores
        const Tensor& x = T(o.in[0]);
        if (x.ndim < 2 || x.shape[x.ndim - 1] != x.shape[x.ndim - 2]) return (why = "causal softmax needs [.., s, s]"), false;
      }
      if (o.kind == TS_OP_DROPOUT && (o.fa[0] < 0 || o.fa[0] >= 1)) return (why = "dropout p"), false;
      return true;
    case TS_OP_ADD:
      if (!need(2, 1)) return false;
      if (!same_shape(T(o.in[0]), T(o.out[0])) || !same_shape(T(o.in[1]), T(o.out[0])))
        return (why = "add shapes"), false;
      return true;
    case TS_OP_LAYERNORM: {
      if (!need(3, 1)) return false;
      const Tensor &x = T(o.in[0]);
      if (x.ndim != 2 || T(o.in[1]).numel != last(x) || T(o.in[2]).numel != last(x) ||
          !same_shape(x, T(o.out[0])))
        return (why = "layernorm shapes"), false;
      if (o.fa.size() < 1) return (why = "layernorm eps"), false;
      return true;
    }
    case TS_OP_ATTN_QK: case TS_OP_ATTN_PV: {
      if (!need(2, 1)) return false;
      if (o.ia.size() < 2) return (why = "attn attrs {heads, seq}"), false;
      int64_t heads = o.ia[0], seq = o.ia[1];
      const Tensor& a = T(o.in[0]);
      const Tensor& b = T(o.in[1]);
      const Tensor& y = T(o.out[0]);
      const Tensor& qk = o.kind == TS_OP_ATTN_QK ? a : b;  // a [T,h] operand
      if (qk.ndim != 2 || qk.shape[1] % heads || qk.shape[0] % seq) return (why = "attn [T,h]"), false;
      int64_t nb = qk.shape[0] / seq;
      const Tensor& s = o.kind == TS_OP_ATTN_QK ? y : a;
      if (s.ndim != 4 || s.shape[0] != nb || s.shape[1] != heads || s.shape[2] != seq || s.shape[3] != seq)
        return (why = "attn [b,a,s,s]"), false;
      if (o.kind == TS_OP_ATTN_QK && (!same_shape(a, b) || o.fa.size() < 1)) return (why = "attn_qk"), false;
      if (o.kind == TS_OP_ATTN_PV && !same_shape(b, y)) return (why = "attn_pv out"), false;
      if ((qk.shape[1] / heads) % 8) return (why = "head dim must be a multiple of 8"), false;
      return true;
    }
    case TS_OP_ATTENTION: {
      if (!need(3, 3)) return false;
      if (o.ia.size() < 3 || o.fa.size() < 2) return (why = "attention attrs {heads, seq, seed} {alpha, p}"), false;
      const int64_t heads = o.ia[0], seq = o.ia[1];
      const Tensor &q = T(o.in[0]), &c = T(o.out[0]), &l = T(o.out[1]);
      if (heads < 1 || seq < 1 || q.ndim != 2 || q.shape[1] % heads || q.shape[0] % seq) return (why = "attention [T,h]"), false;
      if (!same_shape(q, T(o.in[1])) || !same_shape(q, T(o.in[2])) || !same_shape(q, c))
        return (why = "attention Q/K/V/C shapes"), false;
      if (l.ndim != 3 || l.shape[0] * seq != q.shape[0] || l.shape[1] != heads || l.shape[2] != seq ||
          l.dtype != TS_F32)
        return (why = "attention lse must be f32 [b,a,s]"), false;
      if ((q.shape[1] / heads) % 8) return (why = "head dim must be a multiple of 8"), false;
      if (o.fa[1] < 0 || o.fa[1] >= 1) return (why = "attention dropout p"), false;
      const Tensor& mk = T(o.out[2]);
      if (seq % 32 || mk.ndim != 4 || mk.dtype != TS_I32 || mk.shape[0] != l.shape[0] || mk.shape[1] != heads ||
          mk.shape[2] != seq || mk.shape[3] != seq / 32)
        return (why = "attention keep bits must be i32 [b,a,s,s/32] (seq % 32 == 0)"), false;
      return true;
    }
    case TS_OP_EMBED: {
      if (!need(5, 1)) return false;
      const Tensor &ids = T(o.in[0]), &tt = T(o.in[1]), &y = T(o.out[0]);
      if (o.ia.size() < 1) return (why = "embed seq"), false;
      if (ids.dtype != TS_I32 || tt.dtype != TS_I32 || ids.ndim != 1 || !same_shape(ids, tt))
        return (why = "embed ids"), false;
      for (int i = 2; i < 5; ++i)
        if (T(o.in[i]).ndim != 2 || T(o.in[i]).shape[1] != y.shape[1] || T(o.in[i]).kind != TS_PARAM)
          return (why = "embed tables"), false;
      if (y.ndim != 2 || y.shape[0] != ids.shape[0] || T(o.in[3]).shape[0] < o.ia[0])
        return (why = "embed out"), false;
      return true;
    }
    case TS_OP_CLS: {
      if (!need(1, 1)) return false;
      const Tensor &x = T(o.in[0]), &y = T(o.out[0]);
      if (o.ia.size() < 1 || x.ndim != 2 || y.ndim != 2 || x.shape[0] != y.shape[0] * o.ia[0] ||
          x.shape[1] != y.shape[1])
        return (why = "cls shapes"), false;
      return true;
    }
    case TS_OP_CONV2D: {
      if ((o.in.size() != 2 && o.in.size() != 3) || o.out.size() != 1) return (why = "conv2d in/out"), false;
      const Tensor &x = T(o.in[0]), &w = T(o.in[1]), &y = T(o.out[0]);
      if (o.ia.size() < 2 || o.ia[0] < 1 || o.ia[1] < 0) return (why = "conv2d attrs {stride, pad}"), false;
      if (x.ndim != 4 || w.ndim != 4 || y.ndim != 4 || w.kind != TS_PARAM) return (why = "conv2d ranks"), false;
      const int64_t st = o.ia[0], pd = o.ia[1];
      const int64_t P = (x.shape[1] + 2 * pd - w.shape[1]) / st + 1, Q = (x.shape[2] + 2 * pd - w.shape[2]) / st + 1;
      if (w.shape[3] != x.shape[3] || y.shape[0] != x.shape[0] || y.shape[1] != P || y.shape[2] != Q ||
          y.shape[3] != w.shape[0])
        return (why = "conv2d shapes"), false;
      if (o.in.size() == 3 && (T(o.in[2]).numel != w.shape[0] || T(o.in[2]).kind != TS_PARAM))
        return (why = "conv2d bias"), false;
      return true;
    }
    case TS_OP_BATCHNORM: {
      if (!need(3, 1)) return false;
      const Tensor& x = T(o.in[0]);
      if (!same_shape(x, T(o.out[0])) || T(o.in[1]).numel != last(x) || T(o.in[2]).numel != last(x) || o.fa.empty())
        return (why = "batchnorm shapes/eps"), false;
      return true;
    }
    case TS_OP_MAXPOOL: {
      if (!need(1, 1)) return false;
      const Tensor &x = T(o.in[0]), &y = T(o.out[0]);
      if (o.ia.size() < 3 || x.ndim != 4 || y.ndim != 4) return (why = "maxpool attrs/ranks"), false;
      const int64_t k = o.ia[0], st = o.ia[1], pd = o.ia[2];
      if (y.shape[1] != (x.shape[1] + 2 * pd - k) / st + 1 || y.shape[2] != (x.shape[2] + 2 * pd - k) / st + 1 ||
          y.shape[3] != x.shape[3] || y.shape[0] != x.shape[0])
        return (why = "maxpool shapes"), false;
      return true;
    }
    case TS_OP_AVGPOOL: {
      if (!need(1, 1)) return false;
      const Tensor &x = T(o.in[0]), &y = T(o.out[0]);
      if (x.ndim != 4 || y.ndim != 2 || y.shape[0] != x.shape[0] || y.shape[1] != x.shape[3])
        return (why = "avgpool shapes"), false;
      return true;
    }
    case TS_OP_FLATTEN: {
      if (!need(1, 1)) return false;
      const Tensor &x = T(o.in[0]), &y = T(o.out[0]);
      if (y.ndim != 2 || y.shape[0] != x.shape[0] || y.numel != x.numel) return (why = "flatten shapes"), false;
      return true;
    }
    case TS_OP_XENT: {
      if (!need(2, 1)) return false;
      const Tensor &z = T(o.in[0]), &l = T(o.in[1]), &y = T(o.out[0]);
      if (z.ndim != 2 || l.ndim != 1 || l.shape[0] != z.shape[0] || l.dtype != TS_I32 || y.numel != 1 ||
          y.dtype != TS_F32)
        return (why = "xent shapes"), false;
      return true;
    }
  }
  why = "unknown op kind";
  return false;
}

// Saved forward tensors read by each backward op (DESIGN.md §3 "saved").
std::vector<int> saved_of(const Graph& g, const Op& o) {
  std::vector<int> src;
  switch (o.kind) {
    case TS_OP_LINEAR: case TS_OP_GELU: case TS_OP_LAYERNORM: case TS_OP_CONV2D: case TS_OP_BATCHNORM:
    case TS_OP_MAXPOOL:
      src = {o.in[0]};
      break;
    case TS_OP_RELU: case TS_OP_TANH: case TS_OP_SOFTMAX: src = {o.out[0]}; break;
    case TS_OP_ATTN_QK: case TS_OP_ATTN_PV: case TS_OP_EMBED: case TS_OP_XENT: src = {o.in[0], o.in[1]}; break;
    case TS_OP_ATTENTION: src = {o.in[0], o.in[1], o.in[2], o.out[0], o.out[1], o.out[2]}; break;
    default: break;
  }
  std::vector<int> r;
  for (int t : src)
    if (g.t[t].kind != TS_PARAM && std::find(r.begin(), r.end(), t) == r.end()) r.push_back(t);
  return r;
}

}  // namespace

ts_status build_graph(const ts_tensor_desc* td, int nt, const ts_op_desc* od, int no, int samples,
                      int dtype, Graph& g) {
  if (!td || !od || nt <= 0 || no <= 0 || samples <= 0) return set_error("ts_graph_define: bad arguments"), TS_ERR_ARG;
  if (dtype != TS_F32 && dtype != TS_BF16) return set_error("compute dtype must be f32 or bf16"), TS_ERR_ARG;
  g = Graph();
  g.samples = samples;
  g.dtype = dtype;
  g.t.resize(nt);
  for (int i = 0; i < nt; ++i) {
    Tensor& t = g.t[i];
    t.id = i;
    t.dtype = td[i].dtype;
    t.kind = td[i].kind;
    t.ndim = td[i].ndim;
    if (t.ndim < 1 || t.ndim > 6 || t.dtype < 0 || t.dtype > 2 || t.kind < 0 || t.kind > 3)
      return set_error("tensor " + std::to_string(i) + ": bad descriptor"), TS_ERR_ARG;
    t.numel = 1;
    for (int d = 0; d < t.ndim; ++d) {
      t.shape[d] = td[i].shape[d];
      if (t.shape[d] <= 0) return set_error("tensor " + std::to_string(i) + ": bad shape"), TS_ERR_ARG;
      t.numel *= t.shape[d];
    }
    t.bytes = uint64_t(t.numel) * dtype_bytes(t.dtype);
  }
  g.ops.resize(no);
  for (int i = 0; i < no; ++i) {
    Op& o = g.ops[i];
    o.id = i;
    o.kind = od[i].kind;
    if (od[i].n_in < 0 || od[i].n_out < 0 || (od[i].n_in && !od[i].in) || (od[i].n_out && !od[i].out))
      return set_error("op " + std::to_string(i) + ": bad descriptor"), TS_ERR_ARG;
    o.in.assign(od[i].in, od[i].in + od[i].n_in);
    o.out.assign(od[i].out, od[i].out + od[i].n_out);
    if (od[i].n_iattr > 0) o.ia.assign(od[i].iattr, od[i].iattr + od[i].n_iattr);
    if (od[i].n_fattr > 0) o.fa.assign(od[i].fattr, od[i].fattr + od[i].n_fattr);
    for (int x : o.in)
      if (x < 0 || x >= nt) return set_error("op " + std::to_string(i) + ": bad input id"), TS_ERR_GRAPH;
    for (int x : o.out) {
      if (x < 0 || x >= nt) return set_error("op " + std::to_string(i) + ": bad output id"), TS_ERR_GRAPH;
      if (g.t[x].producer >= 0) return set_error("tensor produced twice"), TS_ERR_GRAPH;
      if (g.t[x].kind != TS_ACT) return set_error("op output must be an activation"), TS_ERR_GRAPH;
      g.t[x].producer = i;
    }
  }
  for (auto& o : g.ops) {
    std::string why;
    if (!validate_op(g, o, why))
      return set_error("op " + std::to_string(o.id) + " (kind " + std::to_string(o.kind) + "): " + why),
             TS_ERR_GRAPH;
    for (int x : o.in)
      if (std::find(g.t[x].consumers.begin(), g.t[x].consumers.end(), o.id) == g.t[x].consumers.end())
        g.t[x].consumers.push_back(o.id);
    if (o.kind == TS_OP_XENT) {
      if (g.loss >= 0) return set_error("more than one loss"), TS_ERR_GRAPH;
      g.loss = o.out[0];
      g.t[o.out[0]].is_loss = true;
    }
  }
  if (g.loss < 0) return set_error("graph has no xent loss"), TS_ERR_GRAPH;
  for (auto& t : g.t) {
    std::sort(t.consumers.begin(), t.consumers.end());
    if (t.kind == TS_ACT && t.producer < 0) return set_error("activation without producer"), TS_ERR_GRAPH;
    t.sample = t.kind != TS_PARAM && !t.is_loss;
    if (t.sample) {
      if (t.shape[0] % samples) return set_error("tensor " + std::to_string(t.id) + ": leading dim not a multiple of samples"), TS_ERR_GRAPH;
      t.rows_per_sample = t.shape[0] / samples;
      t.elems_per_sample = t.numel / samples;
    }
    bool aux = false;
    if (t.producer >= 0) {
      const Op& po = g.ops[t.producer];
      for (size_t i = 0; i < po.out.size(); ++i)
        if (po.out[i] == t.id && aux_output(po.kind, int(i))) aux = true;
    }
    if (t.kind == TS_ACT && t.dtype != dtype && !t.is_loss && !aux)
      return set_error("activation dtype must equal the compute dtype"), TS_ERR_GRAPH;
  }
  // needs_grad: params, and everything downstream of one (in definition order
  // fixed-point, so any op order works).
  for (auto& t : g.t) t.needs_grad = t.kind == TS_PARAM;
  for (bool changed = true; changed;) {
    changed = false;
    for (auto& o : g.ops) {
      bool any = false;
      for (int x : o.in) any |= g.t[x].needs_grad;
      if (any)
        for (size_t i = 0; i < o.out.size(); ++i) {
          const int x = o.out[i];
          if (!aux_output(o.kind, int(i)) && !g.t[x].needs_grad) g.t[x].needs_grad = changed = true;
        }
    }
  }
  for (auto& o : g.ops) {
    bool any = false;
    for (int x : o.in) any |= g.t[x].needs_grad;
    o.has_bwd = o.kind == TS_OP_XENT || any;
    o.saved = saved_of(g, o);
  }

  // ---- Alg. 1 ------------------------------------------------------------------
  std::vector<std::vector<int>> preds(no), succ(no);
  for (auto& o : g.ops) {
    for (int x : o.in) {
      int p = g.t[x].producer;
      if (p >= 0 && std::find(preds[o.id].begin(), preds[o.id].end(), p) == preds[o.id].end()) {
        preds[o.id].push_back(p);
        succ[p].push_back(o.id);
      }
    }
  }
  for (auto& s : succ) {
    std::sort(s.begin(), s.end());
    s.erase(std::unique(s.begin(), s.end()), s.end());
  }
  std::vector<int> ref_cnt(no);
  for (int i = 0; i < no; ++i) ref_cnt[i] = (int)preds[i].size();
  g.order.clear();
  // explicit stack instead of recursion (deep chains); visits in the same order
  std::function<void(int)> sched = [&](int layer) {
    std::vector<std::pair<int, size_t>> st{{layer, 0}};
    g.order.push_back(layer);
    while (!st.empty()) {
      auto& [l, idx] = st.back();
      if (idx >= succ[l].size()) {
        st.pop_back();
        continue;
      }
      int nxt = succ[l][idx++];
      if (--ref_cnt[nxt] == 0) {
        g.order.push_back(nxt);
        st.push_back({nxt, 0});
      }
    }
  };
  for (int i = 0; i < no; ++i)
    if (preds[i].empty()) sched(i);
  if ((int)g.order.size() != no) return set_error("graph has a cycle"), TS_ERR_GRAPH;

  // ---- static region: masters | bf16 copies | grads | workspace --------------
  uint64_t off = 0;
  int64_t max1d = 1;
  g.master_off.assign(nt, 0);
  g.copy_off.assign(nt, 0);
  g.grad_off.assign(nt, 0);
  for (auto& t : g.t)
    if (t.kind == TS_PARAM) {
      g.master_off[t.id] = off;
      off += align_up(4 * t.numel);
      if (t.ndim == 1) max1d = std::max<int64_t>(max1d, t.numel);
    }
  for (auto& t : g.t)
    if (t.kind == TS_PARAM && dtype == TS_BF16) {
      g.copy_off[t.id] = off;
      off += align_up(2 * t.numel);
    }
  for (auto& t : g.t)
    if (t.kind == TS_PARAM) {
      g.grad_off[t.id] = off;
      off += align_up(4 * t.numel);
    }
  g.ws_off = off;
  g.ws_bytes = align_up(kWsRows * 2 * uint64_t(max1d) * 4);
  off += g.ws_bytes;
  g.bn_off.assign(no, 0);
  for (auto& o : g.ops)
    if (batch_reduce(o.kind)) {
      g.bn_off[o.id] = off;
      off += align_up(16 * uint64_t(g.t[o.in[0]].shape[g.t[o.in[0]].ndim - 1]));
    }
  g.static_bytes = off;
  return TS_OK;
}

}  // namespace ts
