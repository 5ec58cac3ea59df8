"""NEXT-4 delta-PageRank on the GPU (GUM_DPR; reading #27): the filter hands each activated vertex's
residual over (x += r, push d*r/outdeg), the advance adds the pushes into the destinations' residuals with a
returning fp64 atomic and activates a vertex when its residual crosses eps. The result is an approximation of
x* within the tolerance, so parity is checked against what the definition fixes: x <= x* componentwise,
sum(x* - x) <= tolerance (x* by a sparse linear solve), and the L1 distance to the oracle's BSP rounds <= the
sum of both bounds; the round count matches the oracle's within rounding of the threshold decisions."""
import numpy as np
import pytest

import inputs
import oracle
from tests.gpu_helpers import gpu_run
from tests.test_oracle import dpr_fixpoint

pytestmark = pytest.mark.gpu


def check_dpr(g, tol=1e-6, **kw):
    x, st, _ = gpu_run(g, "dpr", 0, dpr_tolerance=tol, **kw)
    xs, _ = dpr_fixpoint(g)
    xo, _, rounds = oracle.delta_pagerank(g.num_vertices, g.src, g.dst, 0.85, tolerance=tol, return_state=True)
    assert np.all(x <= xs * (1 + 1e-11) + 1e-300), float(np.max(x - xs))
    gap = float((xs - x).sum())
    assert -1e-11 <= gap <= tol + 1e-11, gap
    assert float(np.abs(x - xo).sum()) <= 2 * tol + 1e-11
    assert abs(st.iterations - rounds) <= 2, (st.iterations, rounds)
    assert st.edges_expanded == st.edges_frontier
    return x, st


def test_dpr_hand_graphs():
    n = 64
    cyc = inputs.from_pairs(n, [(i, (i + 1) % n) for i in range(n)])
    x, st = check_dpr(cyc)
    K = 0
    while 0.15 * 0.85 ** K / n > 1e-6 * 0.15 / n:
        K += 1
    assert st.iterations == K and np.allclose(x, (1 - 0.85 ** K) / n, rtol=1e-12)
    star = inputs.from_pairs(21, [(i, 0) for i in range(1, 21)])
    x, st = check_dpr(star, tol=1e-9)
    # (round 2 of the oracle only hands the dangling centre's residual over; on the GPU that is the filter of
    # the second iteration, which queues nothing, so the run ends after one advance)
    assert st.iterations == 1 and abs(x[0] - (0.15 / 21) * (1 + 0.85 * 20)) < 1e-16
    check_dpr(inputs.from_pairs(7, [(0, 1), (1, 2), (2, 0), (3, 3), (3, 3), (5, 6)]))  # pieces, loops, isolated


@pytest.mark.parametrize("P,part", [(1, "seg"), (1, "degree"), (3, "random"), (8, "seg")])
def test_dpr_rmat(P, part):
    g = inputs.rmat(13, 16, seed=81, weighted=False)
    check_dpr(g, num_gpus=P, part=part, seed=4)


@pytest.mark.parametrize("kw", [dict(force_mode="sparse"), dict(force_mode="dense"), dict(num_gpus=4, fsteal=False),
                                dict(num_gpus=4, split_units=True), dict(num_gpus=3, host_loop=True),
                                dict(num_gpus=4, chunk_edges=64), dict(num_gpus=4, osteal_threshold=1 << 30,
                                                                       osteal_edges_per_worker=20000, split_units=True)])
def test_dpr_modes(kw):
    g = inputs.rmat(12, 16, seed=83, weighted=False)
    check_dpr(g, tol=1e-7, **kw)


def test_dpr_long_tail_frontier_shrinks():
    """The active set shrinks over the rounds (the long tail of P:31)."""
    g = inputs.rmat(14, 16, seed=85, weighted=False)
    x, st = check_dpr(g, tol=1e-8, trace=True)
    _, _, tr = gpu_run(g, "dpr", 0, dpr_tolerance=1e-8, trace=True)
    f = [r["frontier_vertices"] for r in tr]
    assert f[0] > 10 * f[-1] and len(f) > 20
