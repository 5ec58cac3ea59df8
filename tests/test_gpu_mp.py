"""Multi-process mode on the GPU: one process per worker (include/gum.h gum_create_mp), the peers'
fragments mapped with CUDA IPC, device-side signal-pad barriers between phases.

The test box has one GPU, so the 2-4 processes share cuda:0 (IPC between processes on one device is the
same mechanism as across NVLink peers; the kernels are time-sliced, which the spin barrier tolerates).
Each rank computes the full result through the peer mappings and compares it with the oracle:
BFS/SSSP/WCC bit-exact, PR rel <= 1e-5 / L1 <= 1e-6, edges expanded == frontier edges (SURVEY.md §8(c)
c-6), for seg/random partitions, FSteal steal-always, and OSteal forced to one owner (the evicted
fragments are then processed by rank 0 through "extended memory").
"""
import pytest

from tests import mp_harness

pytestmark = pytest.mark.gpu


def case_parity(rank, world, scale, part, kw):
    import numpy as np

    import inputs
    import oracle
    from paper_conf_icde_menggltyz23_b200 import dist as gdist
    from tests.gpu_helpers import assert_pr_close

    g = inputs.rmat(scale, 16, seed=scale + world)
    s = inputs.pick_source(g, scale)
    import paper_conf_icde_menggltyz23_b200 as gum

    row_ptr, col, w = gum.build_csr(g.num_vertices, g.src, g.dst, g.w)
    out = {}
    with gdist.mp_context(device=0, **kw) as ctx:
        ctx.load_csr(row_ptr, col, w)
        ctx.partition(part, 5)
        for alg in ("bfs", "sssp", "wcc", "pr"):
            st = ctx.run(alg, s)
            res = ctx.result()
            ref = oracle.run(alg, g, s)
            if alg == "pr":
                assert_pr_close(res, ref)
                ok = True
            else:
                ok = bool(np.array_equal(res, ref))
            out[alg] = dict(ok=ok, conserved=st.edges_expanded == st.edges_frontier, iters=st.iterations,
                            stolen=st.edges_stolen, owners=st.final_owners, remote=st.remote_updates,
                            tail_iters=st.tail_iterations, bodies=st.bodies, osteal_iter=st.osteal_iteration,
                            barriers=list(st.unit_barriers)[:world], last=list(st.unit_last_iter)[:world])
    return out


@pytest.mark.parametrize("world,part,kw", [(2, "random", {}), (3, "seg", {"tail_vertices": 0}),
                                          (4, "random", {"tail_vertices": 0}), (3, "random", {})])
def test_mp_parity(world, part, kw):
    """Default tail threshold (16384) on a 4096-vertex graph: the whole run goes to the tail engine on rank 0
    and the other ranks park in their device-resident loops; tail_vertices=0: every iteration synchronises
    all ranks through the device barrier."""
    res = mp_harness.run("tests.test_gpu_mp", "case_parity", world=world, args=(12, part, kw), timeout=600,
                         hide_gpu=False)
    for r in res:
        for alg, d in r.items():
            assert d["ok"] and d["conserved"], (alg, d)
    for alg in res[0]:
        assert len({r[alg]["iters"] for r in res}) == 1  # every rank left the loop at the same iteration
    if kw.get("tail_vertices") == 0:  # (the tail engine does not count remote updates)
        assert any(r["bfs"]["remote"] > 0 for r in res)


def test_mp_copy_migration():
    """NEXT-3 copy-migration across processes: the owner's foster queues are IPC-mapped for thieves."""
    kw = dict(osteal_migrate=True, tail_vertices=0, osteal_threshold=1 << 30, osteal_edges_per_worker=20000,
              chunk_edges=64)
    res = mp_harness.run("tests.test_gpu_mp", "case_parity", world=3, args=(12, "random", kw), timeout=600,
                         hide_gpu=False)
    for r in res:
        for alg, d in r.items():
            assert d["ok"] and d["conserved"], (alg, d)


def test_mp_forced_stealing_and_osteal():
    """FSteal with 32-edge chunks and no gating, and OSteal shrinking to one owner from the start."""
    kw = dict(chunk_edges=32, osteal_threshold=1 << 40, osteal_edges_per_worker=0)
    res = mp_harness.run("tests.test_gpu_mp", "case_parity", world=2, args=(11, "random", kw), timeout=600,
                         hide_gpu=False)
    for r in res:
        for alg, d in r.items():
            assert d["ok"] and d["conserved"], (alg, d)
    assert res[0]["bfs"]["owners"] == 1
