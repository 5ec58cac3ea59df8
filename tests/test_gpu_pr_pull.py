"""PR pull (the default PR advance, kernels.cu k_pr_pull): merge-path passes over source blocks. Parity with
the oracle's power iteration (rel <= 1e-5, L1 <= 1e-6) across block counts (1 .. 64 passes), worker counts,
partitions, split launch units, rows that span many tiles (in-hubs), empty rows, and agreement with the
push (pr_push=1)."""
import numpy as np
import pytest

import inputs
import oracle
from tests.gpu_helpers import assert_pr_close, check, gpu_run

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("block_bytes", [None, "65536", "8192"])
@pytest.mark.parametrize("P,part", [(1, "seg"), (3, "random"), (8, "seg")])
def test_pr_pull_blocks(monkeypatch, block_bytes, P, part):
    if block_bytes:
        monkeypatch.setenv("GUM_PR_PULL_BLOCK_BYTES", block_bytes)
    g = inputs.rmat(13, 16, seed=41, weighted=False)
    ref = oracle.run("pr", g)
    out, st, _ = check(g, "pr", 0, ref=ref, num_gpus=P, part=part, seed=5)
    assert st.iterations == 20
    assert abs(out.sum() - 1.0) < 1e-9


def test_pr_pull_in_hub_rows_span_tiles(monkeypatch):
    """One vertex with 200K in-edges (its row spans ~100 merge-path tiles in every pass), a second hub
    split over all blocks, many dangling and isolated vertices."""
    monkeypatch.setenv("GUM_PR_PULL_BLOCK_BYTES", "16384")  # 2048-source blocks -> 64 passes at V=2^17
    V = 1 << 17
    rng = np.random.default_rng(7)
    leaves = rng.integers(2, V, 200000)
    src = np.concatenate([leaves, rng.integers(0, V, 300000), np.full(5000, 0), np.arange(2, 40000)])
    dst = np.concatenate([np.zeros(200000, np.int64), rng.integers(0, V, 300000), rng.integers(2, V, 5000),
                          np.ones(40000 - 2, np.int64)])
    g = inputs.EdgeList(V, src.astype(np.uint32), dst.astype(np.uint32), None, "inhub")
    ref = oracle.run("pr", g)
    for P in (1, 2):
        check(g, "pr", 0, ref=ref, num_gpus=P)


def test_pr_pull_matches_push_and_split_units():
    g = inputs.rmat(12, 8, seed=43, weighted=False)
    ref = oracle.run("pr", g)
    pull, _, _ = gpu_run(g, "pr", 0, num_gpus=1)
    push, _, _ = gpu_run(g, "pr", 0, num_gpus=1, pr_push=True)
    assert_pr_close(pull, ref)
    assert_pr_close(push, ref)
    assert np.abs(pull - push).max() / ref.min() < 1e-9
    for kw in (dict(num_gpus=4, split_units=True), dict(num_gpus=2, host_loop=True), dict(num_gpus=3, profile=True)):
        out, st, _ = gpu_run(g, "pr", 0, **kw)
        assert_pr_close(out, ref)
        assert st.edges_expanded == st.edges_frontier


def test_pr_pull_single_vertex_and_no_edges():
    g = inputs.from_pairs(5, [])
    out, _, _ = gpu_run(g, "pr", 0)
    assert np.allclose(out, 0.2, rtol=1e-14)
    g1 = inputs.from_pairs(1, [(0, 0), (0, 0)])
    out, _, _ = gpu_run(g1, "pr", 0)
    assert abs(out[0] - 1.0) < 1e-14
