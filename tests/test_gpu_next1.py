"""NEXT-1: communication reducers of §V-B.

* outer-vertex mirrors with early message aggregation (include/gum.h `mirrors`): PR pushes to other
  fragments aggregate in the worker's local mirror and the owner's finalize pulls them once per iteration;
  BFS sends a vertex at most once per worker ("already sent" bits); SSSP/WCC send only candidates that beat
  the mirror's upper bound of the owner's value;
* hub adjacency caching (P:274 Example 6; `hub_cache`, t4 = `hub_degree`): stolen / inherited frontier
  vertices with out-degree > t4 are expanded from a worker-local copy of their list.

Parity bar as everywhere: BFS/SSSP/WCC bit-exact, PR rel <= 1e-5 / L1 <= 1e-6, conservation
of expanded edges. On top, the counters must show the mechanisms at work, with one exact count: with FSteal
off each chunk is processed by its owner, so PR's aggregated pushes = iterations x cross-fragment edges.
"""
import numpy as np
import pytest

import inputs
import oracle
from tests import mp_harness
from tests.gpu_helpers import assert_pr_close, check, csr_of

pytestmark = pytest.mark.gpu

ALGS = ["bfs", "sssp", "wcc", "pr"]


@pytest.mark.parametrize("alg", ALGS)
@pytest.mark.parametrize("P", [2, 4, 8])
@pytest.mark.parametrize("part", ["seg", "random"])
def test_mirrors_parity(alg, P, part):
    g = inputs.rmat(13, 16, seed=41)
    s = inputs.pick_source(g, 41)
    ref = oracle.run(alg, g, s)
    csr = csr_of(g)
    # (PR: the plain path compared here is the push, whose per-edge remote atomics the mirrors aggregate)
    _, plain, _ = check(g, alg, s, csr=csr, ref=ref, num_gpus=P, part=part, seed=P, tail_vertices=0,
                        pr_push=(alg == "pr"))
    _, st, _ = check(g, alg, s, csr=csr, ref=ref, num_gpus=P, part=part, seed=P, tail_vertices=0, mirrors=True)
    assert st.remote_filtered > 0
    if alg == "pr":
        assert st.remote_updates == 0 and plain.remote_updates > 0  # no per-edge cross-fragment atomics left
        assert st.mirror_flush_bytes == st.iterations * (P - 1) * g.num_vertices * 8


def test_pr_mirror_aggregation_count():
    """FSteal off, seg partition: every cross-fragment edge is aggregated once per iteration."""
    g = inputs.rmat(12, 16, seed=43)
    row_ptr, col, _ = csr_of(g)
    import paper_conf_icde_menggltyz23_b200 as gum

    P = 4
    with gum.Context(num_gpus=P, fsteal=False, mirrors=True, tail_vertices=0) as ctx:
        ctx.load_csr(row_ptr, col)
        ctx.partition("seg", 0)
        b = np.array(ctx.bounds(), dtype=np.int64)
        st = ctx.run("pr")
        x = ctx.result()
    assert_pr_close(x, oracle.run("pr", g))
    src = np.repeat(np.arange(g.num_vertices), np.diff(row_ptr.astype(np.int64)))
    fs = np.searchsorted(b, src, side="right") - 1
    fd = np.searchsorted(b, col.astype(np.int64), side="right") - 1
    cross = int((fs != fd).sum())
    assert st.remote_filtered == st.iterations * cross


@pytest.mark.parametrize("alg", ["bfs", "sssp", "wcc", "pr"])
def test_mirrors_with_stealing_osteal_and_units(alg):
    g = inputs.rmat(13, 8, seed=5, scramble=False)  # hubs at low ids: fragment 0 heavy, stealing happens
    s = inputs.pick_source(g, 5)
    ref = oracle.run(alg, g, s)
    csr = csr_of(g)
    for kw in (dict(chunk_edges=32, num_gpus=4), dict(num_gpus=4, osteal_threshold=1 << 30),
               dict(num_gpus=8, osteal_threshold=1 << 30, osteal_edges_per_worker=1000),
               dict(num_gpus=4, host_loop=True), dict(num_gpus=3, split_units=True),
               dict(num_gpus=4, force_mode="sparse"), dict(num_gpus=4, force_mode="dense"),
               dict(num_gpus=3, tail_vertices=16), dict(num_gpus=4, fsteal="planned")):
        check(g, alg, s, csr=csr, ref=ref, mirrors=True, **kw)


@pytest.mark.parametrize("alg", ["bfs", "sssp", "wcc"])
@pytest.mark.parametrize("t4", [0, 16, 1 << 30])
def test_hub_cache(alg, t4):
    g = inputs.rmat(17, 16, seed=7, scramble=False)  # hubs at low ids: fragment 0 heavy -> others steal
    s = inputs.pick_source(g, 7)
    ref = oracle.run(alg, g, s)
    csr = csr_of(g)
    _, st, _ = check(g, alg, s, csr=csr, ref=ref, num_gpus=4, chunk_edges=64, hub_cache=True, hub_degree=t4,
                     tail_vertices=0)
    assert st.chunks_stolen > 0
    if t4 == 1 << 30:
        assert st.hub_cached_edges == 0
    else:
        assert 0 < st.hub_cached_edges
    if t4 == 0:
        # every non-local expansion reads the copy: stolen edges (no OSteal shrink here) all come from it
        assert st.hub_cached_edges == st.edges_stolen
    # OSteal: worker 0 inherits every fragment ("extended memory") and expands from its copies
    _, st2, _ = check(g, alg, s, csr=csr, ref=ref, num_gpus=4, hub_cache=True, hub_degree=t4, fsteal=False,
                      osteal_threshold=1 << 40, tail_vertices=0)
    assert st2.final_owners == 1
    if t4 == 0:
        assert st2.hub_cached_edges > 0


@pytest.mark.parametrize("alg", ALGS)
def test_mirrors_and_hub_cache_together(alg):
    g = inputs.rmat(13, 16, seed=45)
    s = inputs.pick_source(g, 45)
    ref = oracle.run(alg, g, s)
    csr = csr_of(g)
    for part in ("seg", "random"):
        check(g, alg, s, csr=csr, ref=ref, num_gpus=4, part=part, seed=1, mirrors=True, hub_cache=True,
              hub_degree=8, chunk_edges=128)


def test_mp_mirrors_and_hub_cache():
    """One process per worker: PR mirrors are read by the owner through CUDA IPC; hub copies are local."""
    kw = dict(mirrors=True, hub_cache=True, hub_degree=4, chunk_edges=64)
    res = mp_harness.run("tests.test_gpu_mp", "case_parity", world=3, args=(12, "random", kw), timeout=600,
                         hide_gpu=False)
    for r in res:
        for a, d in r.items():
            assert d["ok"] and d["conserved"], (a, d)
