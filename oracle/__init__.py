"""ORACLE — TEST INFRASTRUCTURE ONLY.

A plain, slow, obviously-correct CPU (numpy fp64 / pure Python) implementation
of what the TSPLIT hot path computes, written from PAPER.md:

  * ops.py     — fp64 forward / VJP of every operator (the unsplit definition;
                 P:L42 "no accuracy loss", P:L471 operators unchanged)
  * net.py     — unsplit forward+backward of a DFG (§II)
  * sim.py     — Alg. 1 schedule, augmented-schedule expansion
                 (Fig. 10), best-fit pool
                  and the resulting allocation trace / peaks
  * execplan.py— executes an expanded plan piece by piece in fp64 (split, swap,
                 memory-centric recompute) to pin plan invariance (T1)
  * brute.py   — brute-force plan enumeration on tiny graphs (T8, T9)

Only `tests/`, `__graft_entry__.smoke()` and `bench.py`'s cpu_baseline /
`--impl reference` legs may import anything under `oracle/`.  The product
(`paper_conf_icde_niemyc22_b200`) never imports it and shares no code with it;
the shared inputs come from `tsinputs` (data only).

Parity unpinned: the planner's *choice* (greedy, not unique) and
its predicted time; the presence of s3 in M_{N-2} (Fig. 3 absent).
"""
