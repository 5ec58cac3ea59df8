"""NEXT-2 FSteal planner: the oracle restatement of Eq. (1) / Alg. 1 pinned by brute force and the paper's
Example 2, and the product's closed-form planner (gum_fsteal_plan, the routine k_control runs) checked
against the oracle LP -- all on CPU."""
import json
import os

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import paper_conf_icde_menggltyz23_b200 as gum
from oracle import planner

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "example2_fsteal.json")


def uniform_costs(n, b):
    return [[1.0 if i == j else b for j in range(n)] for i in range(n)]


def test_example2_golden_oracle():
    g = json.load(open(GOLDEN))
    C = uniform_costs(2, g["remote_cost"])
    z_milp, X_milp = planner.milp_bruteforce(g["loads"], C)
    z_lp, X_lp = planner.lp_relaxation(g["loads"], C)
    assert z_milp == g["expected_z"] and abs(z_lp - g["expected_z"]) < 1e-9
    # the paper's plan (v3 moves) is one of the optimal integer plans (ties exist, e.g. a full swap)
    Xg = np.array(g["expected_X"])
    assert Xg.sum(axis=1).tolist() == g["loads"]
    assert max((np.array(C) * Xg).sum(axis=0)) == z_milp
    rng = planner.carve(g["gpu0_frontier_degrees_v1_v2_v3"], g["expected_X"][0])
    assert rng[0] == tuple(g["expected_carve_gpu0"]["gpu0"]) and rng[1] == tuple(g["expected_carve_gpu0"]["gpu1"])


def test_example2_golden_product():
    g = json.load(open(GOLDEN))
    z, X = gum.fsteal_plan(g["loads"], g["remote_cost"])
    assert abs(z - g["expected_z"]) < 1e-6
    assert np.allclose(X, g["expected_X"], atol=1e-6)


def test_example2_nonuniform_cost_keeps_more_local():
    # "we have to access the neighbors of v3 over NVLink ... the plan of Fig. 3 is not optimal"
    z_lp, X = planner.lp_relaxation([8, 2], uniform_costs(2, 2.0))
    z, Xp = gum.fsteal_plan([8, 2], 2.0)
    assert abs(z - z_lp) < 1e-6 and z > 5.0 and Xp[0, 1] < 3.0


@settings(max_examples=40, deadline=None)
@given(st.lists(st.integers(0, 6), min_size=2, max_size=3), st.sampled_from([1.0, 2.0]))
def test_oracle_lp_lower_bounds_milp(loads, b):
    C = uniform_costs(len(loads), b)
    z_milp, X = planner.milp_bruteforce(loads, C)
    z_lp, _ = planner.lp_relaxation(loads, C)
    assert z_lp <= z_milp + 1e-9
    assert z_milp <= z_lp + max(b, 1.0) * (len(loads) - 1) + 1e-9  # rounding costs at most one edge per thief
    assert [int(r.sum()) for r in X] == list(loads)


@settings(max_examples=80, deadline=None)
@given(st.lists(st.integers(0, 10**9), min_size=1, max_size=8), st.sampled_from([1.0, 1.3, 2.0, 5.0]))
def test_product_planner_matches_oracle_lp(loads, b):
    z, X = gum.fsteal_plan(loads, b)
    z_lp, _ = planner.lp_relaxation(loads, uniform_costs(len(loads), b))
    assert abs(z - z_lp) <= 1e-6 * max(1.0, z_lp)
    assert np.allclose(X.sum(axis=1), loads, rtol=1e-9, atol=1e-3)  # every edge assigned once
    C = np.array(uniform_costs(len(loads), b))
    assert np.all((C * X).sum(axis=0) <= z * (1 + 1e-9) + 1e-3)  # nobody exceeds the makespan
    assert np.all(X >= -1e-9)


def test_product_planner_balanced_loads_no_stealing():
    z, X = gum.fsteal_plan([7, 7, 7], 1.0)
    assert abs(z - 7) < 1e-9 and np.allclose(X, np.diag([7, 7, 7]))


def test_carve_whole_adjacency_lists():
    # P:81 "to avoid splitting the adjacency list ... we select a group of vertices"
    # a vertex goes to the first GPU whose cumulative quota covers the end of its list
    assert planner.carve([4, 4, 4, 4], [6, 10]) == [(0, 1), (1, 4)]
    assert planner.carve([4, 4, 4, 4], [8, 8]) == [(0, 2), (2, 4)]
    assert planner.carve([4, 4, 4, 4], [16, 0]) == [(0, 4), None]


# ------------------------------------------------------------------------------- NEXT-3 OSteal model
GOLDEN3 = os.path.join(os.path.dirname(__file__), "golden", "example3_osteal.json")


def test_example3_golden_oracle():
    g = json.load(open(GOLDEN3))
    C = uniform_costs(2, g["remote_cost"])
    for m, zexp in enumerate(g["expected_z_by_m"], start=1):
        assert planner.osteal_milp_bruteforce(g["loads"], C, m)[0] == zexp
        assert abs(planner.osteal_lp(g["loads"], C, m)[0] - zexp) < 1e-9
    th = g["p_threshold"]
    assert planner.osteal_alg2(g["loads"], C, th - 0.5)[0] == 2
    assert planner.osteal_alg2(g["loads"], C, th)[0] == 1  # tie: the first (smaller) m is kept
    assert planner.osteal_alg2(g["loads"], C, th + 0.5)[0] == 1


def test_example3_golden_product():
    g = json.load(open(GOLDEN3))
    th = g["p_threshold"]
    for p, mexp in ((0.0, 2), (th - 0.5, 2), (th + 0.5, 1), (1e9, 1)):
        m, cost = gum.osteal_plan(g["loads"], g["remote_cost"], p)
        assert m == mexp, (p, m, cost)
        assert np.allclose(cost, [z + p * (k + 1) for k, z in enumerate(g["expected_z_by_m"])], rtol=1e-9)


@settings(max_examples=40, deadline=None)
@given(st.lists(st.integers(0, 3), min_size=2, max_size=3), st.sampled_from([1.0, 2.0]))
def test_osteal_lp_lower_bounds_milp(loads, b):
    C = uniform_costs(len(loads), b)
    for m in range(1, len(loads) + 1):
        z_milp = planner.osteal_milp_bruteforce(loads, C, m)[0]
        z_lp = planner.osteal_lp(loads, C, m)[0]
        assert z_lp <= z_milp + 1e-9
        assert z_milp <= z_lp + b * len(loads) + 1e-9  # integrality gap bounded by one edge per row


@settings(max_examples=60, deadline=None)
@given(st.lists(st.integers(0, 10**7), min_size=1, max_size=8), st.sampled_from([1.0, 1.3, 2.0, 5.0]),
       st.sampled_from([0.0, 1.0, 1e4, 1e6, 1e9]))
def test_product_osteal_matches_oracle_alg2(loads, b, p):
    n = len(loads)
    C = uniform_costs(n, b)
    m_ora, cost_ora = planner.osteal_alg2(loads, C, p)
    m, cost = gum.osteal_plan(loads, b, p)
    scale = max(1.0, max(cost_ora))
    assert np.allclose(cost, cost_ora, atol=1e-6 * scale, rtol=1e-7)
    # the same choice unless two cluster sizes tie within rounding
    if m != m_ora:
        assert abs(cost[m - 1] - cost[m_ora - 1]) <= 1e-6 * scale


def test_osteal_special_cases():
    # m = n is the FSteal plan; m = 1 puts every other fragment's work on worker 0 at the remote cost;
    # more survivors never increase the makespan
    loads = [700, 50, 3000, 0, 12]
    for b in (1.0, 2.5):
        z_f, _ = gum.fsteal_plan(loads, b)
        m, cost = gum.osteal_plan(loads, b, 0.0)
        assert abs(cost[-1] - z_f) < 1e-6 * z_f
        assert abs(cost[0] - (loads[0] + b * sum(loads[1:]))) < 1e-6 * cost[0]
        assert all(cost[i + 1] <= cost[i] + 1e-6 for i in range(len(loads) - 1))
