"""Larger parity cases in the driver's -m gpu run (RMAT-22 EF16: 4.2M vertices, 67M edges; a 2048^2 grid), in
bench.py's launch configurations (DEGREE layout for BFS and PR, tail engine, near-far SSSP, PR at K = 20 with
the OpenMP pull oracle), so the multi-tile filter CTAs, many advance chunks per CTA, several PR source blocks
and the far lists are all exercised against the oracle. (Full BASELINE sizes: tests/test_gpu_full_size.py with
GUM_FULL_SIZE=1, and profiles/round2/parity_full_*.json.)"""
import numpy as np
import pytest

import inputs
import oracle
from tests.gpu_helpers import assert_pr_close, check, csr_of, gpu_run

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def rmat22():
    g = inputs.rmat(22, 16, seed=22)
    return g, csr_of(g), inputs.pick_source(g, 22)


@pytest.mark.parametrize("alg,part", [("bfs", "degree"), ("sssp", "seg"), ("wcc", "seg"), ("bfs", "random")])
def test_rmat22_exact(rmat22, alg, part):
    g, csr, s = rmat22
    check(g, alg, s, csr=csr, part=part, seed=1, tail_vertices=0 if alg == "bfs" else 16384)


def test_rmat22_pr_k20_pull_degree(rmat22, monkeypatch):
    g, csr, _ = rmat22
    monkeypatch.setenv("GUM_PR_PULL_BLOCK_BYTES", str(8 << 20))  # 4 source blocks at V = 2^22
    ref, _ = oracle.pagerank_pull(g.num_vertices, g.src, g.dst, 20, 0.85)
    out, st, _ = gpu_run(g, "pr", 0, csr=csr, part="degree", seed=1)
    assert st.iterations == 20
    assert_pr_close(out, ref)


def test_grid2048_sssp_near_far_far_lists():
    g = inputs.grid(2048, seed=3)
    ref = oracle.run("sssp", g, 0)
    for kw in (dict(sssp_delta=4096), dict(sssp_delta=1024, tail_vertices=0), dict(sssp_delta=600, num_gpus=4,
                                                                                    split_units=True)):
        check(g, "sssp", 0, ref=ref, **kw)
