// Data-parallel gradient buckets: every rank executes
// the same plan, so the point in the augmented schedule after which a parameter's
// gradient is final — the last backward micro-op of the ops that read it (dW merges
// across splits by summation in ascending k) — is the same on every rank.
// Parameters are grouped, in the order their gradients become final, into buckets of
// at least `bucket_bytes`; each bucket is allreduced on the comm stream right after
// its last writer while the remaining backward runs (the overlap of north_star's
// "gradients are allreduced with NCCL over NVLink").  A bucket's parameters are
// merged into contiguous spans of the static gradient region.
#include <algorithm>

#include "core.h"

namespace ts {

std::vector<GradBucket> grad_buckets(const Graph& g, const Expansion& ex, uint64_t bucket_bytes) {
  const int n = g.n();
  std::vector<int> last(n, -1);
  for (size_t i = 0; i < ex.items.size(); ++i) {
    const Item& it = ex.items[i];
    if (it.kind != IT_B) continue;
    for (int x : g.ops[it.op].in)
      if (g.t[x].kind == TS_PARAM) last[x] = int(i);
  }
  std::vector<std::vector<int>> ready(ex.items.size());
  std::vector<int> never;  // params without a gradient writer (stay zero; still reduced, cheaply)
  for (int t = 0; t < n; ++t)
    if (g.t[t].kind == TS_PARAM) {
      if (last[t] >= 0) ready[last[t]].push_back(t);
      else never.push_back(t);
    }
  std::vector<GradBucket> out;
  std::vector<int> pend;
  uint64_t pend_bytes = 0;
  auto emit = [&](int after) {
    if (pend.empty()) return;
    std::sort(pend.begin(), pend.end(), [&](int a, int b) { return g.grad_off[a] < g.grad_off[b]; });
    GradBucket b;
    b.after_item = after;
    for (int t : pend) {
      const uint64_t off = g.grad_off[t], len = align_up(4 * uint64_t(g.t[t].numel));
      if (!b.spans.empty() && b.spans.back().first + b.spans.back().second == off) b.spans.back().second += len;
      else b.spans.push_back({off, len});
    }
    out.push_back(std::move(b));
    pend.clear();
    pend_bytes = 0;
  };
  for (size_t i = 0; i < ex.items.size(); ++i) {
    for (int t : ready[i]) {
      pend.push_back(t);
      pend_bytes += align_up(4 * uint64_t(g.t[t].numel));
    }
    if (pend_bytes >= bucket_bytes) emit(int(i));
  }
  for (int t : never) pend.push_back(t);
  emit(int(ex.items.size()) - 1);
  return out;
}

}  // namespace ts
