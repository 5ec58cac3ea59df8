"""T2/T3 parity: the CUDA path (through the C ABI) vs the CPU oracle on the same seeded inputs.

BFS/SSSP/WCC bit-exact; PR per-vertex relative error <= 1e-5 and L1 <= 1e-6.
Results must not depend on the number of (virtual) workers, the partitioner, FSteal/OSteal or the
frontier mode (§8(c) c-6); conservation of expanded edges is checked on every run.
"""
import numpy as np
import pytest

import inputs
import oracle
from tests.gpu_helpers import check, csr_of, gpu_run

pytestmark = pytest.mark.gpu

ALGS = ["bfs", "sssp", "wcc", "pr"]


def hand_graphs():
    n = 40
    yield "path", inputs.from_pairs(n, [(i, i + 1) for i in range(n - 1)], np.arange(1, n)), 0
    yield "cycle", inputs.from_pairs(n, [(i, (i + 1) % n) for i in range(n)], np.full(n, 3)), 7
    yield "outstar", inputs.from_pairs(n, [(0, i) for i in range(1, n)], np.arange(1, n)), 0
    yield "instar", inputs.from_pairs(n, [(i, 0) for i in range(1, n)], np.arange(1, n)), 0
    yield "pieces", inputs.from_pairs(12, [(0, 1), (0, 1), (1, 1), (1, 2), (4, 5), (5, 4), (2, 0), (9, 10)],
                                      [5, 1, 2, 3, 1, 1, 0, 9]), 0
    yield "isolated", inputs.from_pairs(5, [], []), 2
    yield "single", inputs.from_pairs(1, [(0, 0)], [4]), 0
    yield "grid33", inputs.grid(33, seed=3), 0


@pytest.mark.parametrize("alg", ALGS)
def test_hand_graphs(alg):
    for name, g, s in hand_graphs():
        if g.w is None:
            g.w = np.ones(g.num_edges, np.uint32)
        for P in (1, 3):
            check(g, alg, s, num_gpus=P)


@pytest.mark.parametrize("alg", ALGS)
@pytest.mark.parametrize("scale", [10, 14])
@pytest.mark.parametrize("part", ["seg", "degree"])
def test_rmat_single_worker(alg, scale, part):
    g = inputs.rmat(scale, 16, seed=scale)
    s = inputs.pick_source(g, scale)
    check(g, alg, s, part=part)


def test_c1_bfs_sssp():
    """BASELINE.json configs[0]: RMAT-16 EF16, BFS + SSSP, 1 GPU vs the oracle."""
    g = inputs.make_config("C1")
    s = inputs.pick_source(g, 1)
    csr = csr_of(g)
    check(g, "bfs", s, csr=csr)
    check(g, "sssp", s, csr=csr)
    for alg in ("bfs", "sssp"):  # degree-ordered layout (GUM_PART_DEGREE): same results in original ids
        check(g, alg, s, csr=csr, part="degree")


@pytest.mark.parametrize("alg", ALGS)
@pytest.mark.parametrize("P", [2, 4, 8])
@pytest.mark.parametrize("part", ["seg", "random", "degree"])
@pytest.mark.parametrize("tail", [0, 8192])
def test_virtual_workers_invariance(alg, P, part, tail):
    g = inputs.rmat(13, 16, seed=21)
    s = inputs.pick_source(g, 21)
    ref = oracle.run(alg, g, s)
    csr = csr_of(g)
    check(g, alg, s, csr=csr, ref=ref, num_gpus=P, part=part, seed=P * 7, tail_vertices=tail)


@pytest.mark.parametrize("alg", ["bfs", "sssp", "wcc"])
def test_forced_modes_and_stealing(alg):
    g = inputs.rmat(13, 8, seed=5, scramble=False)  # static skew: hubs at low ids -> fragment 0 heavy
    s = inputs.pick_source(g, 5)
    ref = oracle.run(alg, g, s)
    csr = csr_of(g)
    for kw in (dict(force_mode="sparse"), dict(force_mode="dense"), dict(fsteal=False),
               dict(chunk_edges=32, num_gpus=4), dict(num_gpus=4, osteal_threshold=1 << 30),
               dict(num_gpus=8, osteal_threshold=1 << 30, osteal_edges_per_worker=1000),
               dict(num_gpus=4, host_loop=True), dict(num_gpus=2, use_torch_allocator=True),
               dict(num_gpus=1, tail_vertices=0), dict(num_gpus=3, tail_vertices=16),
               dict(num_gpus=1, tail_vertices=1 << 20), dict(num_gpus=2, profile=True, tail_vertices=64)):
        kw.setdefault("num_gpus", 4)
        out, st, _ = check(g, alg, s, csr=csr, ref=ref, **kw)
        if kw.get("osteal_threshold"):
            assert st.final_owners < kw["num_gpus"]


def test_stealing_happens_and_balances():
    g = inputs.rmat(18, 16, seed=9, scramble=False, weighted=False)  # enough chunks to outlast a worker's CTAs
    s = inputs.pick_source(g, 9)
    csr = csr_of(g)
    ref = oracle.run("bfs", g, s)
    _, st_on, tr_on = check(g, "bfs", s, csr=csr, ref=ref, num_gpus=4, trace=True, chunk_edges=256)
    _, st_off, tr_off = check(g, "bfs", s, csr=csr, ref=ref, num_gpus=4, trace=True, chunk_edges=256, fsteal=False)
    assert st_on.chunks_stolen > 0 and st_off.chunks_stolen == 0
    assert sum(r["frontier_edges"] for r in tr_on) == st_on.edges_frontier
    for r in tr_on:
        assert sum(r["edges_own"]) + sum(r["edges_stolen"]) == r["frontier_edges"]


def test_sssp_unit_weights_equals_bfs():
    g = inputs.rmat(14, 16, seed=3)
    g.w[:] = 1
    s = inputs.pick_source(g, 3)
    csr = csr_of(g)
    a, _, _ = gpu_run(g, "bfs", s, csr=csr)
    b, _, _ = gpu_run(g, "sssp", s, csr=csr)
    assert np.array_equal(a, b)


def test_grid_closed_form_bfs():
    n = 512
    g = inputs.grid(n, unit_weights=True)
    d, _, _ = gpu_run(g, "bfs", 0)
    i, j = np.indices((n, n))
    assert np.array_equal(d.reshape(n, n), (i + j).astype(np.uint32))


def test_pr_torus_uniform():
    g = inputs.torus(128)
    x, st, _ = gpu_run(g, "pr", 0, num_gpus=4)
    assert np.allclose(x, 1.0 / g.num_vertices, rtol=1e-12, atol=0)
    assert st.iterations == 20


def test_errors():
    import paper_conf_icde_menggltyz23_b200 as gum
    g = inputs.from_pairs(3, [(0, 1), (1, 2)], [0xFFFFFFF0, 0x20])
    rp, col, w = csr_of(g)
    with gum.Context() as ctx:
        with pytest.raises(gum.GumError) as e:
            ctx.run("bfs", 0)
        assert e.value.status == gum.GUM_ESTATE
        ctx.load_csr(rp, col, w)
        ctx.partition()
        with pytest.raises(gum.GumError) as e:
            ctx.result()
        assert e.value.status == gum.GUM_ESTATE
        with pytest.raises(gum.GumError) as e:
            ctx.run("bfs", 3)
        assert e.value.status == gum.GUM_ERANGE
        with pytest.raises(gum.GumError) as e:
            ctx.run("sssp", 0)
        assert e.value.status == gum.GUM_ERANGE
        d = ctx.run("bfs", 0)
        assert ctx.result().tolist() == [0, 1, 2]
    with gum.Context() as ctx:
        ctx.load_csr(rp, col, None)
        ctx.partition()
        with pytest.raises(gum.GumError) as e:
            ctx.run("sssp", 0)
        assert e.value.status == gum.GUM_EINVAL
        with pytest.raises(gum.GumError) as e:
            ctx.load_csr(np.array([0, 1, 3, 2], np.uint64), col, None)
        assert e.value.status == gum.GUM_EINVAL
        with pytest.raises(gum.GumError) as e:
            ctx.load_csr(rp, np.array([0, 9], np.uint32), None)
        assert e.value.status == gum.GUM_EINVAL


def test_repeated_runs_reuse_context():
    import paper_conf_icde_menggltyz23_b200 as gum
    g = inputs.rmat(12, 16, seed=2)
    rp, col, w = csr_of(g)
    adj = oracle.Adjacency(g.num_vertices, g.src, g.dst, g.w)
    with gum.Context(num_gpus=2) as ctx:
        ctx.load_csr(rp, col, w)
        ctx.partition("random", 5)
        for s in (0, 17, 100, 4095):
            ctx.run("sssp", s)
            assert np.array_equal(ctx.result(), oracle.sssp(adj, s))
            ctx.run("bfs", s)
            assert np.array_equal(ctx.result(), oracle.bfs(adj, s))
        ctx.run("wcc")
        assert np.array_equal(ctx.result(), oracle.wcc(g.num_vertices, g.src, g.dst))


@pytest.mark.parametrize("alg", ALGS)
def test_split_units_multi_device_path(alg, monkeypatch):
    """GUM_CFG_SPLIT_UNITS: one launch unit (stream + control replica) per worker on one GPU, i.e. the
    multi-device driver (host loop, cross-unit event barriers, redundant per-unit decisions, per-unit
    filter ownership after OSteal) with local instead of P2P pointers."""
    monkeypatch.setenv("GUM_PR_BLOCK_BYTES", "16384")
    g = inputs.rmat(13, 16, seed=41, scramble=False)
    s = inputs.pick_source(g, 41)
    ref = oracle.run(alg, g, s)
    csr = csr_of(g)
    for kw in (dict(num_gpus=2), dict(num_gpus=4, part="random", seed=9),
               dict(num_gpus=4, osteal_threshold=1 << 30, osteal_edges_per_worker=20000),
               dict(num_gpus=3, chunk_edges=64, trace=True)):
        out, st, tr = check(g, alg, s, csr=csr, ref=ref, split_units=True, **kw)
        if tr:
            for r in tr:
                assert sum(r["edges_own"]) + sum(r["edges_stolen"]) == r["frontier_edges"]


@pytest.mark.parametrize("P", [1, 3])
def test_pr_destination_blocked_queue(monkeypatch, P):
    """PR push (pr_push=1): force the destination blocking (8 KiB acc blocks -> many blocks), check parity."""
    monkeypatch.setenv("GUM_PR_BLOCK_BYTES", "8192")
    g = inputs.rmat(13, 16, seed=31, weighted=False)
    ref = oracle.run("pr", g)
    out, st, _ = check(g, "pr", 0, ref=ref, num_gpus=P, part="random" if P > 1 else "seg", seed=3, pr_push=True)
    assert st.vertices_frontier > 20 * np.count_nonzero(np.bincount(g.src, minlength=g.num_vertices))


@pytest.mark.parametrize("delta", [1, 37, 600, 100000])
def test_sssp_near_far_split(delta):
    """Near-far frontier split (sssp_delta > 0): identical distances, fewer re-relaxations on a grid."""
    for g, s in ((inputs.rmat(13, 16, seed=51), None), (inputs.grid(96, seed=3), 0)):
        s = inputs.pick_source(g, 51) if s is None else s
        ref = oracle.run("sssp", g, s)
        csr = csr_of(g)
        base = None
        for kw in (dict(), dict(num_gpus=4, part="random", seed=2), dict(num_gpus=3, split_units=True),
                   dict(force_mode="sparse"), dict(num_gpus=2, osteal_threshold=500)):
            out, st, _ = check(g, "sssp", s, csr=csr, ref=ref, sssp_delta=delta, **kw)
            base = base or st
        if g.name.startswith("grid") and delta <= 600:
            _, st_plain, _ = check(g, "sssp", s, csr=csr, ref=ref)
            assert base.edges_expanded < st_plain.edges_expanded


@pytest.mark.parametrize("alg", ["bfs", "sssp", "wcc"])
@pytest.mark.parametrize("tail", [0, 1, 64, 8192, 16384])
def test_tail_engine_long_chains(alg, tail):
    """High-diameter inputs (the long-tail regime): a 3000-vertex path with shortcuts and a grid; the
    cooperative tail engine must give the oracle's answer whether it never runs, enters/leaves every
    iteration, or runs the whole traversal."""
    n = 3000
    pairs = [(i, i + 1) for i in range(n - 1)] + [(i, i + 37) for i in range(0, n - 37, 97)] + [(n - 1, 5)]
    rng = np.random.default_rng(7)
    w = rng.integers(1, 50, len(pairs))
    for g, s in ((inputs.from_pairs(n, pairs, w), 0), (inputs.grid(80, seed=5), 0)):
        ref = oracle.run(alg, g, s)
        csr = csr_of(g)
        for kw in (dict(), dict(num_gpus=3), dict(num_gpus=2, part="random", seed=4)):
            _, st, _ = check(g, alg, s, csr=csr, ref=ref, tail_vertices=tail, **kw)
            if tail == 8192 and alg != "wcc":
                assert st.tail_iterations > 0
                assert 0 < st.tail_edges <= st.edges_expanded and 0 < st.tail_vertices <= st.vertices_frontier
            if tail == 0:
                assert st.tail_iterations == 0
                assert st.tail_edges == st.tail_vertices == st.tail_activations == 0
            assert st.tail_activations <= st.activations
        if alg == "sssp":
            check(g, alg, s, csr=csr, ref=ref, tail_vertices=tail, sssp_delta=20)


@pytest.mark.parametrize("P", [1, 2])
def test_bfs_propagation_blocking_option(P):
    """pb_block_log2=17 (opt-in): dense BFS iterations bin destination ids and set visited bits in
    shared memory; identical depths (the option is ignored for P > 1)."""
    for g in (inputs.rmat(18, 16, seed=61, weighted=False), inputs.grid(200, unit_weights=True)):
        s = inputs.pick_source(g, 61)
        check(g, "bfs", s, num_gpus=P, pb_block_log2=17)
        check(g, "bfs", s, num_gpus=P, pb_block_log2=17, tail_vertices=0, force_mode="dense")


@pytest.mark.parametrize("alg", ["bfs", "sssp", "wcc", "pr"])
def test_planned_fsteal(alg):
    """fsteal='planned' (NEXT-2): per-iteration Eq. (1) plan + chunk carving instead of the steal queue;
    outputs identical, every chunk processed once, and the executed per-worker loads follow the plan."""
    g = inputs.rmat(16, 16, seed=71, scramble=False)
    s = inputs.pick_source(g, 71)
    ref = oracle.run(alg, g, s)
    csr = csr_of(g)
    for kw in (dict(num_gpus=4), dict(num_gpus=3, fsteal_remote_cost=2.0), dict(num_gpus=2, split_units=True),
               dict(num_gpus=4, tail_vertices=0, chunk_edges=256)):
        _, st, tr = check(g, alg, s, csr=csr, ref=ref, fsteal="planned", trace=True, **kw)
        for r in tr:
            assert sum(r["edges_own"]) + sum(r["edges_stolen"]) == r["frontier_edges"]
    # balance: on the heaviest iteration the executed loads are within a few chunks of each other
    _, st, tr = check(g, "bfs", s, csr=csr, ref=oracle.run("bfs", g, s), fsteal="planned", trace=True,
                      num_gpus=4, tail_vertices=0, chunk_edges=256)
    big = max(tr, key=lambda r: r["frontier_edges"])
    done = [a + b for a, b in zip(big["edges_own"], big["edges_stolen"])]
    assert max(done) - min(done) <= 4 * 256 + 2 * big["frontier_edges"] // 100
    assert st.chunks_stolen > 0


def test_bfs_direction_optimising():
    """NEXT-4 bottom-up BFS iterations (bfs_direction_opt): identical depths on RMAT (where the switch
    fires) and a grid (where it should not), across workers, partitions and launch-unit modes."""
    g = inputs.rmat(17, 16, seed=81, weighted=False)
    s = inputs.pick_source(g, 81)
    ref = oracle.run("bfs", g, s)
    csr = csr_of(g)
    for kw in (dict(), dict(num_gpus=3), dict(num_gpus=4, part="random", seed=6), dict(num_gpus=2, split_units=True),
               dict(tail_vertices=0), dict(num_gpus=2, osteal=False)):
        _, st, _ = check(g, "bfs", s, csr=csr, ref=ref, bfs_direction_opt=True, **kw)
    g2 = inputs.grid(64, unit_weights=True)
    check(g2, "bfs", 0, bfs_direction_opt=True)


@pytest.mark.parametrize("P", [1, 3])
def test_wcc_blocked_first_iteration(monkeypatch, P):
    """WCC iteration 0 on the static destination-blocked symmetric queue (forced with tiny blocks)."""
    monkeypatch.setenv("GUM_WCC_BLOCK_BYTES", "4096")
    g = inputs.rmat(14, 8, seed=91, weighted=False)
    ref = oracle.run("wcc", g)
    csr = csr_of(g)
    blocked = []
    for kw in (dict(), dict(part="random", seed=2), dict(tail_vertices=0), dict(split_units=P > 1),
               dict(force_mode="dense", tail_vertices=0), dict(host_loop=True, trace=True, tail_vertices=0)):
        _, st, tr = check(g, "wcc", 0, csr=csr, ref=ref, num_gpus=P, **kw)
        blocked.append(st.blocked_iterations)
        if tr is not None:  # per-iteration conservation holds in masked blocked passes too
            for r in tr:
                assert sum(r["edges_own"]) + sum(r["edges_stolen"]) == r["frontier_edges"]
    # later dense iterations also ran on the blocked queue (sources masked by the frontier bitmap)
    assert max(blocked) >= 2, blocked


@pytest.mark.parametrize("alg", ALGS)
@pytest.mark.parametrize("p", [1e-9, 2e4, 1e12])
def test_osteal_cost_model(alg, p):
    """NEXT-3: OSteal by Alg. 2 / Eq. (4) (osteal='cost'): outputs unchanged for any p; p -> inf keeps one
    owner, p -> 0 keeps all of them (z(m) is non-increasing in m). (p = 0 itself selects the online estimate,
    tests/test_gpu_units.py test_osteal_online_p.)"""
    g = inputs.rmat(13, 16, seed=33)
    s = inputs.pick_source(g, 33)
    _, st, _ = check(g, alg, s, num_gpus=4, part="random", seed=3, osteal="cost", osteal_sync_edges=p,
                     tail_vertices=0)
    if p == 1e12:
        assert st.final_owners == 1
    if p < 1.0 and alg == "pr":
        assert st.final_owners == 4


@pytest.mark.parametrize("part", ["random", "degree"])
def test_relabel_hub_rows(part):
    """Relabelling moves rows of every length class (thread / warp / CTA-per-row paths of the relabel):
    out-stars with 5000-20000 leaves next to short random rows."""
    rng = np.random.default_rng(3)
    n = 60000
    pairs = [(c, int(x)) for c, k in ((7, 20000), (11, 5000), (40000, 9000)) for x in rng.integers(0, n, k)]
    pairs += [(int(a), int(b)) for a, b in rng.integers(0, n, (200000, 2))]
    g = inputs.from_pairs(n, pairs, rng.integers(1, 256, len(pairs)))
    csr = csr_of(g)
    for alg in ("bfs", "sssp", "wcc"):
        ref = oracle.run(alg, g, 7)
        for P in (1, 3):
            check(g, alg, 7, csr=csr, ref=ref, num_gpus=P, part=part, seed=5)


@pytest.mark.parametrize("alg", ["bfs", "sssp", "wcc"])
def test_tail_engine_append_overflow(alg):
    """One CTA of the tail engine appends more vertices than its shared buffer holds (2048): 40 mid vertices
    of out-degree 250 (below the 256-edge split threshold) discovered together, each with fresh leaves."""
    rng = np.random.default_rng(11)
    mids = list(range(1, 41))
    pairs = [(0, m) for m in mids]
    nxt = 41
    for m in mids:
        pairs += [(m, nxt + j) for j in range(250)]
        nxt += 250
    pairs += [(nxt - 1 - j, j % 41) for j in range(0, 2000, 7)]  # back edges (cycles for WCC/SSSP)
    g = inputs.from_pairs(nxt, pairs, rng.integers(1, 30, len(pairs)))
    ref = oracle.run(alg, g, 0)
    csr = csr_of(g)
    for kw in (dict(), dict(tail_vertices=1 << 16), dict(num_gpus=2, tail_vertices=1 << 16)):
        _, st, _ = check(g, alg, 0, csr=csr, ref=ref, **kw)
