"""ORACLE — test infrastructure only.

Cost formulas of PAPER.md §IV-B written out in the reading SURVEY.md §8(c) fixes:

  Eq. 2 (side condition read as j < i):
      dM_i[s_j, c] = size(s_j),  c in {swap, recompute}
  Eq. 3 (bounds garbled, SURVEY G4 -> reading R5):
      dT_i[s_j, swap] = max(0, S/B_d2h - sum_{u=j+1}^{i-1} (1-Oc_u) T_u)
                      + max(0, S/B_h2d - sum_{u=p}^{q-1}   (1-Oc_u) T_u)
      j = producer position, i = bottleneck, q = first backward consumer,
      p = swap-in start (default q-1, "the previous computation operation")
  Eq. 6 (split across lines, SURVEY G6 -> reading R7):
      dT_i[s_j, (c, p_num, dim)] = (p_num - 1) * dT_i[s_j^(k), c] + dT_split(p_num, dim)
      with micro size S / p_num and dT_split = sum_k T(op on split k) - T(op).
"""

from __future__ import annotations


def eq2_delta_m(size_bytes: int) -> int:
    """Pinned against the simulator's live bytes (test_eq2_delta_m_is_the_size_by_simulation)."""
    return size_bytes


def eq3_swap_cost(size, b_d2h, b_h2d, T, Oc, j, i, p, q):
    """Pinned by T7's special cases (no window / full window / busy link)."""
    fwd_window = sum((1.0 - Oc[u]) * T[u] for u in range(j + 1, i))
    bwd_window = sum((1.0 - Oc[u]) * T[u] for u in range(p, q))
    return max(0.0, size / b_d2h - fwd_window) + max(0.0, size / b_h2d - bwd_window)


def eq6_split_cost(p_num, micro_cost, t_split_sum, t_unsplit):
    """(p_num - 1) x the micro-tensor's swap / recompute cost + dT_split.  The dT_split term
    (c = reside) is pinned against the C++ planner's timeline prediction
    (test_eq6_split_term_equals_the_planner_timeline); the micro-cost term is Eq. 3 / R6
    applied to a piece of size S / p_num."""
    return (p_num - 1) * micro_cost + (t_split_sum - t_unsplit)
