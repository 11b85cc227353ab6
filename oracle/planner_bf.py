"""oracle.planner_bf -- TEST INFRASTRUCTURE ONLY.

Brute-force reference for mu-cuDNN's optimisation problems
(Sec. III).  Everything here enumerates the whole
search space the paper defines and picks the optimum by the definitions; no
dynamic programming, no pruning, no shared code with the product's C++ planner
(paper_conf_cluster_oyamabhm18_b200/csrc/planner.cpp).

Definitions (the scraped paper strips every formula; the readings are
SURVEY.md 8(c) G6-G20, restated in DESIGN.md "Readings"):

* micro-configuration (a, b): algorithm a run on a micro-batch of b samples
  (P:L74).  configuration: a list of micro-configurations whose b sum to the
  mini-batch N; "concatenation" is list concatenation (reading G6).
* timing table: time[a][b] (int64 ns, < 0 = not benchmarked / ineligible) and
  ws[a][b] (bytes) for b = 0..N (column 0 unused) (P:L88 step 1, reading G10).
* WR (Sec. III-B): minimise the total time sum_i time[a_i][b_i] over
  all configurations whose every micro-configuration fits the per-layer
  workspace limit M individually (reading G12).  Canonical answer among ties
  (reading G8/G11): smallest (T, number of parts, parts sorted non-increasing
  and compared lexicographically larger-first, per part (ws, a) smaller-first).
* WD desirable set (Sec. III-C1): a configuration's cost is
  T(C) = sum of times and M(C) = max workspace (reading G13); the desirable set
  is the Pareto front in (T, M): C is kept iff no other configuration C' has
  M(C') <= M(C) and T(C') <= T(C) with (T', M') != (T, M) (reading G15).
* WD ILP (Eq. (1)-(4), reading G16-G18): choose exactly one
  configuration per kernel, minimise the sum of times subject to the sum of
  workspaces (each rounded up to 256 B) <= the total limit.  Canonical answer
  among ties: smallest (sum T, sum M, choice vector lexicographically).
"""
from __future__ import annotations

import itertools
from typing import List, Optional, Sequence, Tuple

ALIGN = 256  # reading G18: each kernel's workspace segment is 256-byte aligned


def align_up(m: int, a: int = ALIGN) -> int:
    return (int(m) + a - 1) // a * a


def _items(n: int, time, ws, cap: Optional[int]):
    """All micro-configurations (a, b) present in the table with ws <= cap,
    ordered by (b descending, ws ascending, a ascending)."""
    items = []
    na = len(time)
    for b in range(1, n + 1):
        for a in range(na):
            t = int(time[a][b])
            if t < 0:
                continue
            m = int(ws[a][b])
            if cap is not None and m > cap:
                continue
            items.append((b, a, t, m))
    items.sort(key=lambda it: (-it[0], it[3], it[1]))
    return items


def enumerate_configurations(n: int, time, ws, cap: Optional[int] = None):
    """Yield every configuration (as a multiset of micro-configurations) whose
    micro-batch sizes sum to n, each micro-configuration present in the table
    and with ws <= cap.  Each multiset is produced exactly once, as a sequence
    non-increasing in the item order of _items().  Yields lists of
    (a, b, t, m)."""
    items = _items(n, time, ws, cap)

    def rec(start: int, remaining: int, acc: list):
        if remaining == 0:
            yield list(acc)
            return
        for i in range(start, len(items)):
            b, a, t, m = items[i]
            if b > remaining:
                continue
            acc.append((a, b, t, m))
            yield from rec(i, remaining - b, acc)
            acc.pop()

    yield from rec(0, n, [])


def _wr_key(cfg):
    T = sum(t for _, _, t, _ in cfg)
    parts = sorted(((b, m, a) for a, b, _, m in cfg), key=lambda x: (-x[0], x[1], x[2]))
    return (T, len(cfg), tuple(-b for b, _, _ in parts), tuple((m, a) for _, m, a in parts))


def wr_bruteforce(n: int, time, ws, limit: int):
    """WR optimum by enumeration of every configuration.
    Returns (total_ns, [(a, b), ...] in non-increasing b) or None if nothing fits."""
    best, best_key = None, None
    for cfg in enumerate_configurations(n, time, ws, cap=limit):
        k = _wr_key(cfg)
        if best_key is None or k < best_key:
            best, best_key = cfg, k
    if best is None:
        return None
    parts = sorted(((b, m, a) for a, b, _, m in best), key=lambda x: (-x[0], x[1], x[2]))
    return best_key[0], [(a, b) for b, _, a in parts]


def pareto(points: Sequence[Tuple[int, int]]) -> List[Tuple[int, int]]:
    """Desirable set (reading G15) of (T, M) points: keep (T, M) iff
    no other point (T', M') != (T, M) has T' <= T and M' <= M.  Written as the
    definition (quadratic), returned sorted by M ascending."""
    uniq = sorted(set((int(t), int(m)) for t, m in points), key=lambda p: (p[1], p[0]))
    keep = []
    for t, m in uniq:
        dominated = any((t2 <= t and m2 <= m) and (t2, m2) != (t, m) for t2, m2 in uniq)
        if not dominated:
            keep.append((t, m))
    return keep


def front_bruteforce(n: int, time, ws, cap: Optional[int] = None):
    """Pareto front over all configurations.  Returns the list of
    (T, M) points sorted by M ascending (T strictly decreasing)."""
    pts = []
    for cfg in enumerate_configurations(n, time, ws, cap=cap):
        pts.append((sum(t for _, _, t, _ in cfg), max(m for _, _, _, m in cfg)))
    return pareto(pts)


def all_configuration_costs(n: int, time, ws, cap: Optional[int] = None):
    """(T, M) of every configuration -- the unpruned ILP variable set."""
    return [(sum(t for _, _, t, _ in cfg), max(m for _, _, _, m in cfg))
            for cfg in enumerate_configurations(n, time, ws, cap=cap)]


def ilp_bruteforce(fronts: Sequence[Sequence[Tuple[int, int]]], total: int):
    """WD 0-1 ILP (Eq. (1)-(4)) by enumerating the product of the
    per-kernel option lists.  fronts[k] = [(t, m), ...].  Returns
    (sum_T, sum_M_aligned, choice tuple, offsets) or None if infeasible."""
    best = None
    for choice in itertools.product(*[range(len(f)) for f in fronts]):
        T = sum(int(fronts[k][c][0]) for k, c in enumerate(choice))
        M = sum(align_up(fronts[k][c][1]) for k, c in enumerate(choice))
        if M > total:
            continue
        key = (T, M, choice)
        if best is None or key < best:
            best = key
    if best is None:
        return None
    T, M, choice = best
    offsets, off = [], 0
    for k, c in enumerate(choice):
        offsets.append(off)
        off += align_up(fronts[k][c][1])
    return T, M, choice, offsets


def ilp_scipy(fronts: Sequence[Sequence[Tuple[int, int]]], total: int):
    """The same ILP handed to a library MILP solver (scipy.optimize.milp / HiGHS)
    exactly as Eq. (1)-(4) state it: binary x_kc, one per kernel, knapsack
    budget.  Returns the optimal objective (int) or None if infeasible."""
    import numpy as np
    from scipy.optimize import Bounds, LinearConstraint, milp

    nvar = sum(len(f) for f in fronts)
    c = np.zeros(nvar)
    mem = np.zeros(nvar)
    A_eq = np.zeros((len(fronts), nvar))
    j = 0
    for k, f in enumerate(fronts):
        for (t, m) in f:
            c[j] = float(t)
            mem[j] = float(align_up(m))
            A_eq[k, j] = 1.0
            j += 1
    cons = [LinearConstraint(A_eq, 1, 1), LinearConstraint(mem[None, :], -np.inf, float(total))]
    res = milp(c, constraints=cons, integrality=np.ones(nvar), bounds=Bounds(0, 1),
               options={"mip_rel_gap": 0.0})
    if res.status != 0:
        return None
    x = np.round(res.x).astype(int)
    ts = [int(t) for f in fronts for (t, _) in f]
    return sum(t for t, xv in zip(ts, x) if xv)
