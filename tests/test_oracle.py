"""T0: pin the CPU oracle to things other than itself.

Pins: closed forms (path, cycle, star, grid i+j, torus 1/V, star PR recurrence), library routines
(scipy.sparse.csgraph shortest_path / dijkstra / connected_components, networkx.pagerank), and
brute force on tiny graphs (boolean reachability powers, Floyd-Warshall, dense-matrix PR).
Each pin is chosen so that a plausible mistake (dropped term, wrong sign/index, transposed operand,
off-by-one) fails at least one of them.
"""
import networkx as nx
import numpy as np
import pytest
import scipy.sparse as sp
from hypothesis import given, settings, strategies as st
from scipy.sparse import csgraph

import inputs
import oracle

INF = oracle.INF


# ----------------------------------------------------------------------------- helpers (brute force)
def random_graph(rng, V, E, wmax=255, wmin=1):
    src = rng.integers(0, V, E, dtype=np.int64).astype(np.uint32)
    dst = rng.integers(0, V, E, dtype=np.int64).astype(np.uint32)
    w = rng.integers(wmin, wmax + 1, E, dtype=np.int64).astype(np.uint32)
    return inputs.EdgeList(V, src, dst, w)


def brute_bfs(g, s):
    """Boolean reachability powers: depth[v] = min k with (e_s A^k)[v] != 0 via dense matrix products."""
    V = g.num_vertices
    A = np.zeros((V, V), dtype=np.int64)
    A[g.src.astype(np.int64), g.dst.astype(np.int64)] = 1
    depth = np.full(V, INF, dtype=np.uint64)
    reach = np.zeros(V, dtype=np.int64)
    reach[s] = 1
    depth[s] = 0
    for k in range(1, V + 1):
        reach = ((reach @ A) > 0).astype(np.int64)
        newly = (reach > 0) & (depth == INF)
        depth[newly] = k
    return depth.astype(np.uint32)


def brute_sssp_fw(g, s):
    """Floyd-Warshall over the min-weight simple graph (parallel edges -> min), zero weights allowed."""
    V = g.num_vertices
    big = np.iinfo(np.int64).max // 4
    D = np.full((V, V), big, dtype=np.int64)
    np.fill_diagonal(D, 0)
    for u, v, w in zip(g.src.tolist(), g.dst.tolist(), g.w.tolist()):
        if u != v:
            D[u, v] = min(D[u, v], w)
    for k in range(V):
        D = np.minimum(D, D[:, k:k + 1] + D[k:k + 1, :])
    d = D[s]
    out = np.where(d >= big, INF, d).astype(np.uint32)
    return out


def brute_bellman_ford(g, s):
    """V*E Bellman-Ford on the raw multigraph."""
    V = g.num_vertices
    dist = [None] * V
    dist[s] = 0
    for _ in range(V):
        changed = False
        for u, v, w in zip(g.src.tolist(), g.dst.tolist(), g.w.tolist()):
            if dist[u] is not None and (dist[v] is None or dist[u] + w < dist[v]):
                dist[v] = dist[u] + w
                changed = True
        if not changed:
            break
    return np.array([INF if d is None else d for d in dist], dtype=np.uint32)


def scipy_min_weight_csr(g):
    """Parallel edges reduced by min (scipy would sum duplicates), self-loops dropped."""
    key = g.src.astype(np.int64) * g.num_vertices + g.dst.astype(np.int64)
    order = np.lexsort((g.w, key))
    key_s, w_s = key[order], g.w[order]
    first = np.ones(len(key_s), dtype=bool)
    first[1:] = key_s[1:] != key_s[:-1]
    key_u, w_u = key_s[first], w_s[first]
    r, c = key_u // g.num_vertices, key_u % g.num_vertices
    keep = r != c
    return sp.csr_matrix((w_u[keep].astype(np.float64), (r[keep], c[keep])),
                         shape=(g.num_vertices, g.num_vertices))


def to_u32_dist(d):
    return np.where(np.isinf(d), INF, d).astype(np.uint64).astype(np.uint32)


# ----------------------------------------------------------------------------- c-1 BFS
def test_bfs_path():
    n = 50
    g = inputs.from_pairs(n, [(i, i + 1) for i in range(n - 1)])
    assert np.array_equal(oracle.run("bfs", g, 0), np.arange(n, dtype=np.uint32))
    d = oracle.run("bfs", g, 10)
    assert np.all(d[:10] == INF) and np.array_equal(d[10:], np.arange(n - 10))


def test_bfs_directed_cycle():
    n, s = 37, 5
    g = inputs.from_pairs(n, [(i, (i + 1) % n) for i in range(n)])
    d = oracle.run("bfs", g, s)
    for i in range(n):
        assert d[(s + i) % n] == i


def test_bfs_out_star_and_in_star():
    n = 20
    out_star = inputs.from_pairs(n, [(0, i) for i in range(1, n)])
    d = oracle.run("bfs", out_star, 0)
    assert d[0] == 0 and np.all(d[1:] == 1)
    in_star = inputs.from_pairs(n, [(i, 0) for i in range(1, n)])
    d = oracle.run("bfs", in_star, 0)
    assert d[0] == 0 and np.all(d[1:] == INF)


def test_bfs_grid_closed_form():
    n = 64
    g = inputs.grid(n)
    d = oracle.run("bfs", g, 0).reshape(n, n)
    i, j = np.indices((n, n))
    assert np.array_equal(d, (i + j).astype(np.uint32))


def test_bfs_unreachable_pieces_selfloops_parallel():
    g = inputs.from_pairs(8, [(0, 1), (0, 1), (1, 1), (1, 2), (4, 5), (5, 4), (2, 0)])
    d = oracle.run("bfs", g, 0)
    assert d.tolist() == [0, 1, 2, INF, INF, INF, INF, INF]


@settings(max_examples=40, deadline=None)
@given(st.integers(1, 40), st.integers(0, 200), st.integers(0, 2**32 - 1))
def test_bfs_vs_brute_force(V, E, seed):
    rng = np.random.default_rng(seed)
    g = random_graph(rng, V, E)
    s = int(rng.integers(0, V))
    assert np.array_equal(oracle.run("bfs", g, s), brute_bfs(g, s))


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_bfs_vs_scipy(seed):
    rng = np.random.default_rng(seed)
    g = random_graph(rng, 3000, 9000)
    s = int(rng.integers(0, 3000))
    ref = csgraph.shortest_path(scipy_min_weight_csr(g), method="D", unweighted=True, indices=s)
    assert np.array_equal(oracle.run("bfs", g, s), to_u32_dist(ref))


def test_bfs_rmat_vs_scipy():
    g = inputs.rmat(12, 8, seed=4)
    s = inputs.pick_source(g, 4)
    ref = csgraph.shortest_path(scipy_min_weight_csr(g), method="D", unweighted=True, indices=s)
    assert np.array_equal(oracle.run("bfs", g, s), to_u32_dist(ref))


# ----------------------------------------------------------------------------- c-2 SSSP
def test_sssp_unit_weights_equals_bfs():
    g = inputs.rmat(12, 8, seed=9)
    g.w[:] = 1
    s = inputs.pick_source(g, 9)
    assert np.array_equal(oracle.run("sssp", g, s), oracle.run("bfs", g, s))


def test_sssp_weighted_path_prefix_sums():
    n = 40
    w = np.arange(1, n, dtype=np.uint32) * 7
    g = inputs.from_pairs(n, [(i, i + 1) for i in range(n - 1)], w)
    d = oracle.run("sssp", g, 0)
    assert np.array_equal(d, np.concatenate([[0], np.cumsum(w)]).astype(np.uint32))


def test_sssp_unit_grid_closed_form():
    n = 48
    g = inputs.grid(n, unit_weights=True)
    d = oracle.run("sssp", g, 0).reshape(n, n)
    i, j = np.indices((n, n))
    assert np.array_equal(d, (i + j).astype(np.uint32))


def test_sssp_prefers_cheaper_longer_path():
    # 0->2 costs 10 directly, 0->1->2 costs 2+3 = 5
    g = inputs.from_pairs(3, [(0, 2), (0, 1), (1, 2)], [10, 2, 3])
    assert oracle.run("sssp", g, 0).tolist() == [0, 2, 5]


def test_sssp_range_error():
    g = inputs.from_pairs(3, [(0, 1), (1, 2)], [0xFFFFFFF0, 0x20])
    with pytest.raises(oracle.OracleRangeError):
        oracle.run("sssp", g, 0)


@settings(max_examples=40, deadline=None)
@given(st.integers(1, 30), st.integers(0, 150), st.integers(0, 2**32 - 1))
def test_sssp_vs_floyd_warshall_zero_weights_allowed(V, E, seed):
    rng = np.random.default_rng(seed)
    g = random_graph(rng, V, E, wmax=20, wmin=0)
    s = int(rng.integers(0, V))
    d = oracle.run("sssp", g, s)
    assert np.array_equal(d, brute_sssp_fw(g, s))
    assert np.array_equal(d, brute_bellman_ford(g, s))


@pytest.mark.parametrize("seed", [1, 2])
def test_sssp_vs_scipy_dijkstra(seed):
    g = inputs.rmat(13, 8, seed=seed)
    s = inputs.pick_source(g, seed)
    ref = csgraph.dijkstra(scipy_min_weight_csr(g), indices=s)
    assert np.array_equal(oracle.run("sssp", g, s), to_u32_dist(ref))


def test_sssp_grid_vs_scipy():
    g = inputs.grid(60, seed=3)
    ref = csgraph.dijkstra(scipy_min_weight_csr(g), indices=0)
    assert np.array_equal(oracle.run("sssp", g, 0), to_u32_dist(ref))


# ----------------------------------------------------------------------------- c-3 WCC
def check_wcc_against_scipy(g):
    lab = oracle.run("wcc", g)
    V = g.num_vertices
    A = sp.csr_matrix((np.ones(g.num_edges), (g.src.astype(np.int64), g.dst.astype(np.int64))), shape=(V, V))
    ncomp, comp = csgraph.connected_components(A, directed=True, connection="weak")
    mins = np.full(ncomp, V, dtype=np.int64)
    np.minimum.at(mins, comp, np.arange(V))
    assert np.array_equal(lab, mins[comp].astype(np.uint32))
    # invariants
    assert np.all(lab <= np.arange(V))
    assert np.array_equal(lab[lab], lab)
    assert np.all(lab[g.src] == lab[g.dst])
    assert len(np.unique(lab)) == ncomp


def test_wcc_disjoint_cycles_isolated():
    pairs = []
    for base, n in [(0, 5), (5, 7), (20, 3)]:
        pairs += [(base + (i + 1) % n, base + i) for i in range(n)]  # reversed direction: weak only
    g = inputs.from_pairs(30, pairs)
    lab = oracle.run("wcc", g)
    exp = list(range(30))
    for base, n in [(0, 5), (5, 7), (20, 3)]:
        for i in range(n):
            exp[base + i] = base
    assert lab.tolist() == exp


def test_wcc_grid_single_component():
    assert np.all(oracle.run("wcc", inputs.grid(30)) == 0)


def test_wcc_direction_ignored():
    # 3 -> 1 <- 2 : one weak component with min 1; 0 isolated
    g = inputs.from_pairs(4, [(3, 1), (2, 1)])
    assert oracle.run("wcc", g).tolist() == [0, 1, 1, 1]


@settings(max_examples=40, deadline=None)
@given(st.integers(1, 60), st.integers(0, 80), st.integers(0, 2**32 - 1))
def test_wcc_vs_scipy_random(V, E, seed):
    rng = np.random.default_rng(seed)
    check_wcc_against_scipy(random_graph(rng, V, E))


def test_wcc_rmat_vs_scipy():
    check_wcc_against_scipy(inputs.rmat(13, 2, seed=6, weighted=False))


# ----------------------------------------------------------------------------- c-4 PageRank
def dense_pagerank(g, K, d):
    """Matrix form: x_{k+1} = (1-d)/V + d (P^T x_k + (dangling . x_k)/V), P row-stochastic (multiplicity)."""
    V = g.num_vertices
    A = np.zeros((V, V))
    np.add.at(A, (g.src.astype(np.int64), g.dst.astype(np.int64)), 1.0)
    out = A.sum(axis=1)
    P = np.divide(A, out[:, None], out=np.zeros_like(A), where=out[:, None] > 0)
    dang = (out == 0).astype(np.float64)
    x = np.full(V, 1.0 / V)
    for _ in range(K):
        x = (1 - d) / V + d * (P.T @ x + (dang @ x) / V)
    return x


def test_pr_mass_conservation_every_k():
    g = inputs.rmat(11, 8, seed=2, weighted=False)
    for K in (0, 1, 2, 7, 20):
        x = oracle.pagerank(g.num_vertices, g.src, g.dst, K, 0.85)
        assert abs(x.sum() - 1.0) < 1e-12


def test_pr_regular_torus_uniform():
    g = inputs.torus(64)
    x = oracle.pagerank(g.num_vertices, g.src, g.dst, 20, 0.85)
    assert np.allclose(x, 1.0 / g.num_vertices, rtol=1e-13, atol=0)


def test_pr_directed_cycle_uniform():
    n = 101
    g = inputs.from_pairs(n, [(i, (i + 1) % n) for i in range(n)])
    x = oracle.pagerank(n, g.src, g.dst, 20, 0.85)
    assert np.allclose(x, 1.0 / n, rtol=1e-13, atol=0)


def test_pr_out_star_two_variable_recurrence():
    n = 9  # centre 0 -> leaves 1..n ; leaves dangling
    V = n + 1
    g = inputs.from_pairs(V, [(0, i) for i in range(1, V)])
    d, K = 0.85, 20
    xc, xl = 1.0 / V, 1.0 / V
    for _ in range(K):
        D = n * xl
        xc, xl = (1 - d) / V + d * (D / V), (1 - d) / V + d * (xc / n + D / V)
    x = oracle.pagerank(V, g.src, g.dst, K, d)
    assert abs(x[0] - xc) < 1e-15 and np.allclose(x[1:], xl, rtol=1e-14)


def test_pr_parallel_edges_count_multiplicity():
    # 0 -> 1 twice, 0 -> 2 once: node 1 receives 2/3 of 0's mass
    g = inputs.from_pairs(3, [(0, 1), (0, 1), (0, 2), (1, 0), (2, 0)])
    x = oracle.pagerank(3, g.src, g.dst, 1, 0.85)
    x0 = 1 / 3
    assert abs(x[1] - (0.15 / 3 + 0.85 * (2 / 3) * x0)) < 1e-15
    assert abs(x[2] - (0.15 / 3 + 0.85 * (1 / 3) * x0)) < 1e-15


@settings(max_examples=30, deadline=None)
@given(st.integers(1, 50), st.integers(0, 200), st.integers(0, 2**32 - 1), st.integers(0, 25))
def test_pr_vs_dense_matrix(V, E, seed, K):
    rng = np.random.default_rng(seed)
    g = random_graph(rng, V, E)
    x = oracle.pagerank(V, g.src, g.dst, K, 0.85)
    ref = dense_pagerank(g, K, 0.85)
    assert np.allclose(x, ref, rtol=1e-12, atol=1e-15)


def test_pr_vs_dense_matrix_rmat_2048():
    g = inputs.rmat(11, 8, seed=3, weighted=False)
    x = oracle.pagerank(g.num_vertices, g.src, g.dst, 20, 0.85)
    assert np.allclose(x, dense_pagerank(g, 20, 0.85), rtol=1e-11, atol=0)


def test_pr_fixpoint_vs_networkx():
    g = inputs.rmat(10, 8, seed=12, weighted=False)
    G = nx.MultiDiGraph()
    G.add_nodes_from(range(g.num_vertices))
    G.add_edges_from(zip(g.src.tolist(), g.dst.tolist()))
    ref = nx.pagerank(G, alpha=0.85, tol=1e-15, max_iter=1000)
    ref = np.array([ref[i] for i in range(g.num_vertices)])
    x = oracle.pagerank(g.num_vertices, g.src, g.dst, 200, 0.85)
    assert np.allclose(x, ref, rtol=1e-9, atol=0)


def test_pr_residuals_decrease_geometrically():
    g = inputs.rmat(11, 8, seed=7, weighted=False)
    _, r = oracle.pagerank(g.num_vertices, g.src, g.dst, 20, 0.85, return_residuals=True)
    assert np.all(r[1:] <= r[:-1] * 0.85 + 1e-15)


# ---- OpenMP pull variant: pinned to the serial power iteration and to the matrix form
def test_pr_pull_equals_serial_rmat16_k20():
    g = inputs.rmat(16, 16, seed=1, weighted=False)
    x, r, used = oracle.pagerank_pull(g.num_vertices, g.src, g.dst, 20, 0.85, threads=4, return_residuals=True)
    xs, rs = oracle.pagerank(g.num_vertices, g.src, g.dst, 20, 0.85, return_residuals=True)
    assert used == 4
    # same terms summed in the same per-vertex order (stable in-edge sort): bit-identical x_K
    assert np.array_equal(x, xs)
    assert float(np.max(np.abs(x - xs) / xs)) <= 1e-13
    assert np.allclose(r, rs, rtol=1e-10, atol=0)


@settings(max_examples=20, deadline=None)
@given(st.integers(1, 40), st.integers(0, 160), st.integers(0, 2**32 - 1), st.integers(0, 22), st.integers(1, 5))
def test_pr_pull_vs_dense_matrix(V, E, seed, K, T):
    rng = np.random.default_rng(seed)
    g = random_graph(rng, V, E)
    x, used = oracle.pagerank_pull(V, g.src, g.dst, K, 0.85, threads=T)
    assert used == T
    assert np.allclose(x, dense_pagerank(g, K, 0.85), rtol=1e-12, atol=1e-15)


def test_pr_pull_torus_uniform():
    g = inputs.torus(48)
    x, _ = oracle.pagerank_pull(g.num_vertices, g.src, g.dst, 20, 0.85, threads=3)
    assert np.allclose(x, 1.0 / g.num_vertices, rtol=1e-13, atol=0)
    assert abs(x.sum() - 1.0) < 1e-12


# ---- NEXT-4 delta-PageRank (reading #27): pinned to the target fixpoint x* (a linear solve, not the
# push), closed forms and networkx
def dpr_fixpoint(g, d=0.85):
    """x* = (I - d P^T)^{-1} (1-d)/V with P = D^{-1} A (multiplicity counted; dangling rows zero)."""
    V = g.num_vertices
    A = sp.coo_matrix((np.ones(g.num_edges), (g.src.astype(np.int64), g.dst.astype(np.int64))), shape=(V, V)).tocsr()
    out = np.asarray(A.sum(axis=1)).ravel()
    inv = np.divide(1.0, out, out=np.zeros_like(out), where=out > 0)
    P = sp.diags(inv) @ A
    M = sp.identity(V, format="csc") - d * P.T.tocsc()
    import scipy.sparse.linalg as spla
    return spla.spsolve(M, np.full(V, (1 - d) / V)), M


def check_dpr_bounds(g, x, r, eps, d=0.85):
    xs, M = dpr_fixpoint(g, d)
    import scipy.sparse.linalg as spla
    V = g.num_vertices
    assert np.all(r <= eps)  # converged: no residual above the threshold
    assert np.all(x <= xs * (1 + 1e-12) + 1e-300)  # x approaches x* from below
    gap = float((xs - x).sum())
    assert -1e-12 <= gap <= V * eps / (1 - d) + 1e-12
    # bookkeeping identity x + (I - d P^T)^{-1} r = x*
    assert np.allclose(x + spla.spsolve(M, r), xs, rtol=1e-10, atol=1e-15)


def test_dpr_directed_cycle_closed_form():
    n, d = 50, 0.85
    g = inputs.from_pairs(n, [(i, (i + 1) % n) for i in range(n)])
    eps = oracle.dpr_epsilon(n, 1e-6)
    x, r, K = oracle.delta_pagerank(n, g.src, g.dst, d, eps=eps, return_state=True)
    # every vertex holds (1-d) d^k / V in round k; it is active while that exceeds eps
    K_ref = 0
    while (1 - d) * d ** K_ref / n > eps:
        K_ref += 1
    assert K == K_ref
    assert np.allclose(x, (1 - d ** K_ref) / n, rtol=1e-12, atol=0)


def test_dpr_in_star_exact():
    n, d = 20, 0.85  # leaves 1..n -> centre 0 (the centre is dangling)
    V = n + 1
    g = inputs.from_pairs(V, [(i, 0) for i in range(1, V)])
    x, r, K = oracle.delta_pagerank(V, g.src, g.dst, d, tolerance=1e-9, return_state=True)
    t = (1 - d) / V
    assert K == 2
    assert np.allclose(x[1:], t, rtol=1e-15) and abs(x[0] - (t + d * n * t)) < 1e-16
    assert np.all(r == 0)


@settings(max_examples=30, deadline=None)
@given(st.integers(1, 60), st.integers(0, 300), st.integers(0, 2**32 - 1), st.sampled_from([1e-3, 1e-6, 1e-9]))
def test_dpr_bounds_random(V, E, seed, tol):
    rng = np.random.default_rng(seed)
    g = random_graph(rng, V, E)
    eps = oracle.dpr_epsilon(V, tol)
    x, r, _ = oracle.delta_pagerank(V, g.src, g.dst, 0.85, eps=eps, return_state=True)
    check_dpr_bounds(g, x, r, eps)


def test_dpr_rmat_bounds_and_networkx():
    g = inputs.rmat(11, 8, seed=21, weighted=False)
    eps = oracle.dpr_epsilon(g.num_vertices, 1e-7)
    x, r, K = oracle.delta_pagerank(g.num_vertices, g.src, g.dst, 0.85, eps=eps, return_state=True)
    check_dpr_bounds(g, x, r, eps)
    assert K > 20  # the frontier-driven rounds have a long tail
    # no dangling vertex (a self-loop on every vertex): x* is the normalised PageRank networkx computes
    V = 512
    pairs = [(v, v) for v in range(V)] + list(zip(*np.random.default_rng(3).integers(0, V, (2, 3000)).tolist()))
    h = inputs.from_pairs(V, pairs)
    xh = oracle.delta_pagerank(V, h.src, h.dst, 0.85, tolerance=1e-9)
    G = nx.MultiDiGraph()
    G.add_nodes_from(range(V))
    G.add_edges_from(zip(h.src.tolist(), h.dst.tolist()))
    ref = nx.pagerank(G, alpha=0.85, tol=1e-15, max_iter=1000)
    ref = np.array([ref[i] for i in range(V)])
    assert float(np.abs(xh - ref).sum()) <= 1e-9 + 1e-12
