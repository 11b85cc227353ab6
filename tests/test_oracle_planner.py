"""Pins for the brute-force planner oracle (oracle/planner_bf.py) -- CPU only.

Checked against things other than itself:
* enumeration counts equal the known partition numbers (one algorithm: p(n);
  two algorithms: OEIS A000712) -- a dropped or duplicated configuration fails;
* closed forms: linear time -> undivided; convex time -> all ones; the paper's
  worked examples P:L74 and Fig. 5 (tests/golden/, scaled, closed-form optima);
* the desirable-set definition on a hand example (Fig. 7 concept);
* the ILP against a library MILP solver (scipy.optimize.milp / HiGHS);
* the paper's stated identities: WR's C(B) is on the WD front;
  pruning never loses the ILP optimum (P:L129-141 proof); `undivided` equals
  plain per-layer selection; WD with the same total memory is never
  worse than WR.
"""
import itertools
import json
import os

import numpy as np
import pytest

from oracle import planner_bf as bf
from synthetic import random_timing_table

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")

PARTITIONS = [1, 1, 2, 3, 5, 7, 11, 15, 22, 30, 42, 56, 77]          # p(n), n = 0..12
TWO_COLOR = [1, 2, 5, 10, 20, 36, 65, 110, 185, 300, 481]            # A000712, n = 0..10


def _full_table(n, na, t=1):
    time = np.full((na, n + 1), t, dtype=np.int64)
    time[:, 0] = -1
    return time, np.zeros((na, n + 1), dtype=np.uint64)


@pytest.mark.parametrize("n", range(1, 13))
def test_enumeration_count_one_algorithm(n):
    time, ws = _full_table(n, 1)
    assert sum(1 for _ in bf.enumerate_configurations(n, time, ws)) == PARTITIONS[n]


@pytest.mark.parametrize("n", range(1, 11))
def test_enumeration_count_two_algorithms(n):
    time, ws = _full_table(n, 2)
    assert sum(1 for _ in bf.enumerate_configurations(n, time, ws)) == TWO_COLOR[n]


def test_linear_time_gives_undivided():
    n = 10
    time = np.array([[-1] + [50 + 7 * b for b in range(1, n + 1)]], dtype=np.int64)
    ws = np.zeros_like(time, dtype=np.uint64)
    T, plan = bf.wr_bruteforce(n, time, ws, limit=0)
    assert plan == [(0, n)] and T == 50 + 7 * n


def test_convex_time_gives_all_ones():
    n = 9
    time = np.array([[-1] + [b * b for b in range(1, n + 1)]], dtype=np.int64)
    ws = np.zeros_like(time, dtype=np.uint64)
    T, plan = bf.wr_bruteforce(n, time, ws, limit=0)
    assert plan == [(0, 1)] * n and T == n


def test_workspace_limit_is_per_micro_config():
    """Reading G12: each micro-configuration must fit M on its own (WR reuses
    one segment sequentially)."""
    n = 8
    time = np.array([[-1] + [100 * b for b in range(1, n + 1)],
                     [-1] + [10 * b for b in range(1, n + 1)]], dtype=np.int64)
    ws = np.array([[0] * (n + 1), [0] + [1000 * b for b in range(1, n + 1)]], dtype=np.uint64)
    T, plan = bf.wr_bruteforce(n, time, ws, limit=3000)
    assert plan == [(1, 3), (1, 3), (1, 2)] and T == 80
    assert bf.wr_bruteforce(n, time, ws, limit=10 ** 9)[1] == [(1, 8)]


def test_golden_fig5_repeated_micro_batch():
    g = json.load(open(os.path.join(GOLDEN, "fig5_repeated_micro_batch.json")))
    n, na = g["n"], g["n_algos"]
    time = np.full((na, n + 1), -1, dtype=np.int64)
    for a in g["rule"]["linear_algos"]:
        for b in range(1, n + 1):
            time[a, b] = g["rule"]["t_linear"][0] + g["rule"]["t_linear"][1] * b
    sp = g["rule"]["special"]
    time[sp["algo"], sp["b"]] = sp["t"]
    ws = np.zeros((na, n + 1), dtype=np.uint64)
    T, plan = bf.wr_bruteforce(n, time, ws, limit=g["ws_limit"])
    assert T == g["expect_total_ns"]
    assert plan == [tuple(p) for p in g["expect_plan"]]


def test_p74_example_scaled():
    """P:L74 shape at N=16: algorithm 1 fits only b <= 4, per-part overhead,
    closed-form optimum 4 x (1,4) (golden p74 file states the N=256 version)."""
    n = 16
    time = np.array([[-1] + [40 * b for b in range(1, n + 1)],
                     [-1] + [10 + 10 * b for b in range(1, n + 1)]], dtype=np.int64)
    ws = np.array([[0] * (n + 1), [0] + [1000 * b for b in range(1, n + 1)]], dtype=np.uint64)
    T, plan = bf.wr_bruteforce(n, time, ws, limit=4000)
    assert plan == [(1, 4)] * 4 and T == 200


def test_no_feasible_plan():
    n = 4
    time = np.array([[-1, 5, 5, 5, 5]], dtype=np.int64)
    ws = np.array([[0, 10, 20, 30, 40]], dtype=np.uint64)
    assert bf.wr_bruteforce(n, time, ws, limit=5) is None


def test_undivided_equals_per_layer_selection():
    """with only b = N benchmarked, WR returns the fastest algorithm
    that fits (cuDNN's own per-layer choice)."""
    for seed in range(20):
        n = 6
        time, ws = random_timing_table(n, 3, seed=seed, sizes={n}, p_absent=0.0)
        limit = int(np.median(ws[:, n]))
        res = bf.wr_bruteforce(n, time, ws, limit)
        fit = [(int(time[a, n]), int(ws[a, n]), a) for a in range(3) if int(ws[a, n]) <= limit]
        t, m, a = min(fit)
        assert res == (t, [(a, n)])


def test_pareto_hand_example():
    """Fig. 7 concept: a point is undesirable iff another is at least
    as fast with no more workspace."""
    pts = [(10, 0), (8, 5), (9, 5), (8, 6), (3, 20), (3, 25), (5, 10), (6, 12), (10, 0)]
    assert bf.pareto(pts) == [(10, 0), (8, 5), (5, 10), (3, 20)]


@pytest.mark.parametrize("seed", range(25))
def test_wr_optimum_is_on_front(seed):
    """WR's C(B) is an element of the WD set, and for every limit M the
    fastest front point within M equals the WR optimum (invariant I3)."""
    n = 7
    time, ws = random_timing_table(n, 3, seed=seed, ties=(seed % 2 == 0))
    front = bf.front_bruteforce(n, time, ws)
    limits = sorted(set(int(v) for v in ws.ravel())) + [10 ** 12]
    for M in limits:
        wr = bf.wr_bruteforce(n, time, ws, M)
        fit = [t for t, m in front if m <= M]
        if wr is None:
            assert not fit
        else:
            assert min(fit) == wr[0]


@pytest.mark.parametrize("seed", range(20))
def test_ilp_bruteforce_matches_scipy_milp(seed):
    g = np.random.default_rng(seed)
    K = int(g.integers(1, 5))
    fronts = []
    for _ in range(K):
        L = int(g.integers(1, 5))
        ms = sorted(g.integers(0, 5000, size=L).tolist())
        ts = sorted(g.integers(1, 10000, size=L).tolist(), reverse=True)
        fronts.append(list(zip(ts, ms)))
    total = int(g.integers(0, 5000 * K))
    got = bf.ilp_bruteforce(fronts, total)
    ref = bf.ilp_scipy(fronts, total)
    if ref is None:
        assert got is None
    else:
        assert got is not None and got[0] == ref


def test_ilp_budget_sweep_closed_forms():
    fronts = [[(100, 0), (60, 1000), (40, 5000)], [(80, 0), (30, 3000)], [(50, 256)]]
    fastest = sum(min(t for t, _ in f) for f in fronts)
    big = sum(bf.align_up(max(m for _, m in f)) for f in fronts)
    assert bf.ilp_bruteforce(fronts, big)[0] == fastest
    minimal = sum(bf.align_up(min(m for _, m in f)) for f in fronts)
    res = bf.ilp_bruteforce(fronts, minimal)
    assert res[0] == 100 + 80 + 50 and res[2] == (0, 0, 0)
    assert bf.ilp_bruteforce(fronts, minimal - 1) is None
    # offsets are the running sum of aligned segments (reading G18)
    T, M, choice, off = bf.ilp_bruteforce(fronts, 1024 + 3072 + 256)
    assert choice == (1, 1, 0) and off == [0, 1024, 1024 + 3072] and T == 60 + 30 + 50


@pytest.mark.parametrize("seed", range(12))
def test_pruning_keeps_ilp_optimum(seed):
    """the ILP over desirable (Pareto) sets has the same optimum as
    over all configurations (invariant I5)."""
    n = 5
    K = 3
    tables = [random_timing_table(n, 2, seed=100 * seed + k, ties=True) for k in range(K)]
    full = [bf.all_configuration_costs(n, t, w) for t, w in tables]
    pruned = [bf.front_bruteforce(n, t, w) for t, w in tables]
    allm = sorted(set(bf.align_up(m) for f in full for _, m in f))
    for total in [0, 256, 512, 1024, 2048, 4096]:
        a = bf.ilp_bruteforce(full, total)
        b = bf.ilp_bruteforce(pruned, total)
        assert (a is None) == (b is None)
        if a is not None:
            assert a[0] == b[0] and a[1] == b[1]
    assert allm is not None


@pytest.mark.parametrize("seed", range(10))
def test_wd_never_worse_than_wr_at_same_total(seed):
    """P:L263/P:L269 (invariant I4): T_WD(K*M) <= sum_k T_WR,k(M)."""
    n, K = 6, 3
    tables = [random_timing_table(n, 3, seed=50 * seed + k) for k in range(K)]
    for M in [0, 256, 4096, 1 << 18, 1 << 20]:
        wr = [bf.wr_bruteforce(n, t, w, M) for t, w in tables]
        if any(r is None for r in wr):
            continue
        fronts = [bf.front_bruteforce(n, t, w) for t, w in tables]
        # each WR segment rounded up to 256 B (reading G18), as WD will do
        wd = bf.ilp_bruteforce(fronts, K * bf.align_up(M))
        assert wd is not None and wd[0] <= sum(r[0] for r in wr)
