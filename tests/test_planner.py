"""The product's C++ planner (csrc/planner.cpp via the C ABI) against the
brute-force oracle (oracle/planner_bf.py) -- bit-exact, CPU only."""
import json
import os

import numpy as np
import pytest

import paper_conf_cluster_oyamabhm18_b200 as mu
from oracle import planner_bf as bf
from synthetic import random_timing_table

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _limits(ws):
    return sorted(set(int(v) for v in ws.ravel()))[:6] + [1 << 40]


@pytest.mark.parametrize("seed", range(60))
def test_wr_dp_equals_bruteforce(seed):
    n = 3 + seed % 8
    time, ws = random_timing_table(n, 3, seed=seed, ties=(seed % 3 == 0))
    for M in _limits(ws):
        ref = bf.wr_bruteforce(n, time, ws, M)
        if ref is None:
            with pytest.raises(mu.MucuError) as e:
                mu.plan_wr(n, time, ws, M)
            assert e.value.status == 3  # INSUFFICIENT_WORKSPACE
        else:
            assert mu.plan_wr(n, time, ws, M) == ref


@pytest.mark.parametrize("policy_sizes", ["pow2", "undivided"])
def test_wr_dp_with_policy_subsets(policy_sizes):
    n = 12
    sizes = {1, 2, 4, 8, 12} if policy_sizes == "pow2" else {12}
    for seed in range(15):
        time, ws = random_timing_table(n, 3, seed=seed, sizes=sizes, p_absent=0.1)
        for M in _limits(ws):
            ref = bf.wr_bruteforce(n, time, ws, M)
            if ref is not None:
                assert mu.plan_wr(n, time, ws, M) == ref


def test_golden_fig5():
    g = json.load(open(os.path.join(GOLDEN, "fig5_repeated_micro_batch.json")))
    n = g["n"]
    time = np.full((3, n + 1), -1, np.int64)
    # The ABI has 3 algorithm slots; map the fixture's "algorithm 4" to slot 2
    # and its equal linear algorithms 0-3 to slot 0 (slot 1 a duplicate).
    for a in (0, 1):
        for b in range(1, n + 1):
            time[a, b] = 100 + 100 * b
    time[2, 6] = 300
    ws = np.zeros((3, n + 1), np.uint64)
    T, plan = mu.plan_wr(n, time, ws, 0)
    assert T == g["expect_total_ns"]
    assert plan == [(2, 6), (2, 6), (2, 6), (0, 2)]


def test_golden_p74_full_n256():
    g = json.load(open(os.path.join(GOLDEN, "p74_four_equal_micro_batches.json")))
    n = g["n"]
    time = np.full((3, n + 1), -1, np.int64)
    ws = np.zeros((3, n + 1), np.uint64)
    for b in range(1, n + 1):
        time[0, b] = 40 * b
        time[1, b] = 10 + 10 * b
        ws[1, b] = 1000 * b
    T, plan = mu.plan_wr(n, time, ws, g["ws_limit"])
    assert T == g["expect_total_ns"] and plan == [tuple(p) for p in g["expect_plan"]]


def test_closed_forms_n256():
    n = 256
    lin = np.full((3, n + 1), -1, np.int64)
    lin[0, 1:] = 1000 + 7 * np.arange(1, n + 1)
    ws = np.zeros((3, n + 1), np.uint64)
    assert mu.plan_wr(n, lin, ws, 0) == (1000 + 7 * n, [(0, n)])
    cvx = np.full((3, n + 1), -1, np.int64)
    cvx[1, 1:] = np.arange(1, n + 1) ** 2
    assert mu.plan_wr(n, cvx, ws, 0) == (n, [(1, 1)] * n)


@pytest.mark.parametrize("seed", range(40))
def test_pareto_front_equals_bruteforce(seed):
    n = 3 + seed % 6
    time, ws = random_timing_table(n, 3, seed=1000 + seed, ties=(seed % 2 == 0))
    ref = bf.front_bruteforce(n, time, ws)
    got = mu.pareto_front(n, time, ws)
    assert [(t, m) for t, m, _ in got] == ref
    for t, m, plan in got:  # each returned plan is a valid configuration with that cost
        assert sum(b for _, b in plan) == n
        assert sum(int(time[a, b]) for a, b in plan) == t
        assert max(int(ws[a, b]) for a, b in plan) == m
        assert all(time[a, b] >= 0 for a, b in plan)


def test_pareto_front_cap():
    n = 6
    time, ws = random_timing_table(n, 3, seed=77)
    cap = int(np.median(ws[ws > 0]))
    ref = bf.front_bruteforce(n, time, ws, cap=cap)
    got = mu.pareto_front(n, time, ws, cap)
    assert [(t, m) for t, m, _ in got] == ref


@pytest.mark.parametrize("seed", range(40))
def test_solve_wd_equals_bruteforce(seed):
    g = np.random.default_rng(seed)
    K = int(g.integers(1, 6))
    fronts = []
    for _ in range(K):
        L = int(g.integers(1, 5))
        if seed % 2:
            f = [(int(g.integers(1, 6)) * 10, int(g.integers(0, 4)) * 256) for _ in range(L)]  # many ties
        else:
            f = [(int(g.integers(1, 10000)), int(g.integers(0, 6000))) for _ in range(L)]
        fronts.append(f)
    for total in [0, 300, 1000, 3000, 8000, 20000]:
        ref = bf.ilp_bruteforce(fronts, total)
        if ref is None:
            with pytest.raises(mu.MucuError) as e:
                mu.solve_wd(fronts, total)
            assert e.value.status == 4  # INFEASIBLE
        else:
            T, choice, off = mu.solve_wd(fronts, total)
            assert (T, tuple(choice), off) == (ref[0], ref[2], ref[3])


@pytest.mark.parametrize("K", [15, 60, 159])
def test_solve_wd_matches_scipy_milp_large(K):
    """Network-sized instances (AlexNet 15, ResNet-18 60, ResNet-50 159 kernels)."""
    g = np.random.default_rng(K)
    fronts = []
    for _ in range(K):
        L = int(g.integers(1, 8))
        ms = sorted(int(v) for v in g.integers(0, 64 << 20, size=L))
        ts = sorted((int(v) for v in g.integers(10_000, 5_000_000, size=L)), reverse=True)
        fronts.append(list(zip(ts, ms)))
    for frac in [0.05, 0.25, 0.6]:
        total = int(frac * sum(max(m for _, m in f) for f in fronts))
        ref = bf.ilp_scipy(fronts, total)
        if ref is None:
            continue
        T, choice, off = mu.solve_wd(fronts, total)
        assert T == ref
        used = sum(bf.align_up(fronts[k][c][1]) for k, c in enumerate(choice))
        assert used <= total and T == sum(fronts[k][c][0] for k, c in enumerate(choice))


def test_network_plan_from_tables_matches_bruteforce():
    """Whole WD pipeline (fronts + ILP) from stored tables (P:L159 offline DB)."""
    n = 5
    net = mu.Network()
    tables = []
    for k in range(3):
        d = mu.desc(n, 16, 8, 8, 16, 3, 3, 1, 1, mu.MATH_F32)
        net.add(d, k % 3)
        tables.append(random_timing_table(n, 3, seed=500 + k, ties=True))
    total = 2048
    net.plan_from_tables(total, tables)
    fronts = [bf.front_bruteforce(n, t, w, cap=total) for t, w in tables]
    ref = bf.ilp_bruteforce(fronts, total)
    got_T = 0
    for k in range(3):
        plan, off, nbytes, t = net.get(k)
        assert off == ref[3][k] and nbytes == bf.align_up(fronts[k][ref[2][k]][1])
        assert sum(b for _, b in plan) == n
        got_T += t
    assert got_T == ref[0]
