"""Device-resident multi-unit loop: one CUDA graph per launch unit
(GUM_CFG_SPLIT_UNITS on one GPU runs the same code path as one device per worker), device barriers over the
member units only, OSteal eviction = the unit leaves the barriers and parks in its graph ("GPU1 will
not participate in synchronization anymore"), give-back wakes it, and the tail engine (OSteal's
m'=1) runs on unit 0 across every fragment. Results must equal the oracle's; the per-unit barrier-arrival
counters show that evicted units stop arriving; host launches do not depend on the iteration count."""
import numpy as np
import pytest

import inputs
import oracle
from tests.gpu_helpers import check, csr_of

pytestmark = pytest.mark.gpu

ALGS = ["bfs", "sssp", "wcc", "pr"]


@pytest.mark.parametrize("alg", ["bfs", "sssp", "wcc"])
@pytest.mark.parametrize("P", [2, 4])
def test_evicted_units_stop_arriving(alg, P):
    """OSteal to one owner from iteration 0 (threshold above any frontier, no tail engine): units 1..P-1 leave
    at the first phase-A barrier after the eviction and arrive at no later barrier."""
    g = inputs.grid(64, seed=5)
    ref = oracle.run(alg, g, 0)
    _, st, _ = check(g, alg, 0, ref=ref, num_gpus=P, split_units=True, osteal_threshold=1 << 40,
                     osteal_edges_per_worker=0, tail_vertices=0)
    assert st.final_owners == 1
    assert st.unit_barriers[0] >= st.iterations  # unit 0 kept synchronising (with itself: no-op barriers)
    for u in range(1, P):
        assert st.unit_last_iter[u] <= st.osteal_iteration + 1, (u, st.unit_last_iter, st.osteal_iteration)
        assert st.unit_barriers[u] <= 2 * (st.osteal_iteration + 1) + 1, st.unit_barriers


@pytest.mark.parametrize("alg", ["bfs", "sssp", "wcc"])
def test_tail_engine_across_units(alg):
    """A high-diameter grid whose frontier stays below the tail threshold: control hands the run to the tail
    engine on unit 0 (every fragment through peer pointers) and the other units park."""
    g = inputs.grid(96, seed=6)
    ref = oracle.run(alg, g, 0)
    for P in (2, 4):
        _, st, _ = check(g, alg, 0, ref=ref, num_gpus=P, split_units=True, tail_vertices=16384)
        assert st.tail_iterations > 0
        assert st.final_owners == 1
        for u in range(1, P):
            assert st.unit_last_iter[u] <= st.osteal_iteration + 1


def blob_chain_blob(scale_a=10, chain=40, scale_b=14, seed=3):
    """RMAT blob A -> a 40-vertex chain -> a symmetrised RMAT blob B (entered at its vertex 0)."""
    a = inputs.rmat(scale_a, 8, seed=seed, weighted=False)
    b = inputs.rmat(scale_b, 8, seed=seed + 1, weighted=False)
    Va, Vb = a.num_vertices, b.num_vertices
    c0, b0 = Va, Va + chain
    V = b0 + Vb
    chain_src = np.concatenate([[0], np.arange(c0, c0 + chain)])
    chain_dst = np.concatenate([np.arange(c0, c0 + chain), [b0]])
    src = np.concatenate([a.src, chain_src, b.src + b0, b.dst + b0]).astype(np.uint32)
    dst = np.concatenate([a.dst, chain_dst, b.dst + b0, b.src + b0]).astype(np.uint32)
    w = np.random.default_rng(seed).integers(1, 256, src.shape[0]).astype(np.uint32)
    return inputs.EdgeList(V, src, dst, w, "blob-chain-blob")


@pytest.mark.parametrize("alg", ["bfs", "sssp"])
def test_give_back_wakes_parked_units(alg):
    """The frontier shrinks to a chain (tail engine on unit 0, units 1..3 parked), then explodes in the second
    blob: the engine hands back, ownership is given back and the parked units are woken (they rejoin and finish
    the run with unit 0)."""
    g = blob_chain_blob()
    ref = oracle.run(alg, g, 0)
    _, st, _ = check(g, alg, 0, ref=ref, num_gpus=4, split_units=True, tail_vertices=32)
    assert st.tail_iterations > 0
    # the parked units were woken and kept synchronising after the tail phase (an evicted unit that is never
    # woken arrives at <= 3 barriers), and they were members at the end of the run
    assert min(st.unit_barriers) >= 8, st.unit_barriers


def test_host_launches_independent_of_iterations():
    """Device-resident loop: the host launches init kernels and one graph per unit, whatever the iteration
    count (a 40-vertex path vs a 400-vertex path)."""
    counts = []
    for n in (40, 400):
        g = inputs.from_pairs(n, [(i, i + 1) for i in range(n - 1)])
        out, st, _ = check(g, "bfs", 0, ref=oracle.run("bfs", g, 0), num_gpus=4, split_units=True, tail_vertices=0)
        assert st.iterations >= n - 1
        counts.append(st.host_launches)
    assert counts[0] == counts[1], counts


@pytest.mark.parametrize("alg", ALGS)
def test_units_match_host_loop_and_oracle(alg):
    g = inputs.rmat(13, 16, seed=51, scramble=False)
    s = inputs.pick_source(g, 51)
    ref = oracle.run(alg, g, s)
    csr = csr_of(g)
    for kw in (dict(num_gpus=3), dict(num_gpus=4, part="random", seed=2), dict(num_gpus=4, host_loop=True),
               dict(num_gpus=8, osteal_threshold=1 << 30, osteal_edges_per_worker=30000)):
        check(g, alg, s, csr=csr, ref=ref, split_units=True, **kw)


@pytest.mark.parametrize("alg", ["bfs", "sssp", "wcc"])
def test_units_repeated_runs_race_check(alg):
    """Shared fragment state touched by several units' kernels in the same iteration is where the device loop
    can race (e.g. a late control clearing the tail engine's list counters): repeat the multi-unit variants
    (tail engine on unit 0 with every other unit parked, shrink/grow with stealing, give-back) 12 times."""
    g = inputs.rmat(12, 16, seed=61, scramble=False)
    s = inputs.pick_source(g, 61)
    ref = oracle.run(alg, g, s)
    csr = csr_of(g)
    gb = blob_chain_blob(9, 30, 12, seed=5)
    ref_gb = oracle.run(alg, gb, 0)
    csr_gb = csr_of(gb)
    for _ in range(12):
        check(g, alg, s, csr=csr, ref=ref, num_gpus=8, split_units=True, osteal_threshold=1 << 30,
              osteal_edges_per_worker=30000)
        check(g, alg, s, csr=csr, ref=ref, num_gpus=5, split_units=True, tail_vertices=0, chunk_edges=64)
        check(gb, alg, 0, csr=csr_gb, ref=ref_gb, num_gpus=4, split_units=True, tail_vertices=32)


@pytest.mark.parametrize("alg", ["bfs", "sssp", "wcc"])
@pytest.mark.parametrize("kw", [dict(num_gpus=4, split_units=True), dict(num_gpus=4), dict(num_gpus=3, split_units=True,
                                                                                          part="random", seed=3)])
def test_osteal_online_p(alg, kw):
    """NEXT-3: p of Eq. (4) estimated during the run from previous iterations: osteal='cost' with
    osteal_sync_edges=0 measures each iteration's synchronisation time against its advance time per edge;
    outputs stay exact whatever owner sets it picks."""
    g = inputs.grid(128, seed=9)
    ref = oracle.run(alg, g, 0)
    _, st, _ = check(g, alg, 0, ref=ref, osteal="cost", osteal_sync_edges=0.0, tail_vertices=0, **kw)
    assert st.osteal_p_samples > 0
    assert 0.0 < st.osteal_p < 1e12


@pytest.mark.parametrize("alg", ["bfs", "sssp", "wcc"])
@pytest.mark.parametrize("kw", [dict(num_gpus=4, split_units=True), dict(num_gpus=4), dict(num_gpus=8, part="random",
                                                                                         seed=5, split_units=True)])
def test_copy_migration_of_evicted_frontiers(alg, kw):
    """NEXT-3 copy-migration (osteal_migrate=1): once OSteal evicts a GPU, its fragment's frontier
    queue is generated in a foster buffer on the new owner and expanded from there; results stay exact and the
    counters show the migrated queue entries (with and without the tail engine, with stealing)."""
    g = inputs.rmat(12, 16, seed=71, scramble=False)
    s = inputs.pick_source(g, 71)
    ref = oracle.run(alg, g, s)
    csr = csr_of(g)
    for extra in (dict(tail_vertices=0, osteal_threshold=1 << 30, osteal_edges_per_worker=40000),
                  dict(tail_vertices=0, osteal="cost", osteal_sync_edges=0.0, chunk_edges=64),
                  dict(tail_vertices=64, osteal_threshold=1 << 30, osteal_edges_per_worker=40000)):
        _, st, _ = check(g, alg, s, csr=csr, ref=ref, osteal_migrate=True, **extra, **kw)
        if "osteal_threshold" in extra and st.final_owners < kw["num_gpus"]:
            assert st.migrated_queue_entries > 0, st
