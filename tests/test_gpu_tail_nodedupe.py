"""Tail engine with and without next-list dedupe bits (GUM_TAIL_NODEDUPE, read once per process, hence the
subprocesses). Default (1): an improvement is decided by the returning atomicMin alone, so a list may hold a
vertex twice; the hand-back to the regular path deduplicates. GUM_TAIL_SLACK=0 shrinks the lists' spare
capacity to nothing, so lists that outgrow V overflow into the frontier bitmap and the engine hands back a
dense frontier (tail_put). Results must be the oracle's (min-fixpoints), with conservation, on
high-diameter inputs where the engine runs most iterations, with and without near-far, one and several
workers, and the engine entering/leaving every iteration."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import sys
sys.path.insert(0, ROOT)
import numpy as np
import inputs, oracle
from tests.gpu_helpers import check, csr_of
n = 3000
pairs = [(i, i + 1) for i in range(n - 1)] + [(i, i + 37) for i in range(0, n - 37, 97)] + [(n - 1, 5)]
w = np.random.default_rng(7).integers(1, 50, len(pairs))
graphs = [(inputs.from_pairs(n, pairs, w), 0), (inputs.grid(96, seed=5), 0), (inputs.grid(256, seed=9), 0)]
g = inputs.rmat(14, 16, seed=17)
graphs.append((g, inputs.pick_source(g, 17)))
ovf = 0
for alg in ("sssp", "wcc", "bfs"):
    for gi, (g, s) in enumerate(graphs):
        ref = oracle.run(alg, g, s)
        csr = csr_of(g)
        for kw in (dict(tail_vertices=8192), dict(tail_vertices=1), dict(tail_vertices=8192, num_gpus=3),
                   dict(tail_vertices=8192, num_gpus=2, part="random", seed=4), dict(tail_vertices=1 << 22)):
            _, st, _ = check(g, alg, s, csr=csr, ref=ref, **kw)
            ovf += st.tail_overflows
        if alg == "sssp":
            check(g, alg, s, csr=csr, ref=ref, tail_vertices=16384, sssp_delta=64)
            _, st, _ = check(g, alg, s, csr=csr, ref=ref, tail_vertices=16384, sssp_delta=1024)
            if gi in (1, 2):
                assert st.tail_iterations > 0
        print("ok", alg, gi, flush=True)
print("overflows", ovf, flush=True)
"""


@pytest.mark.parametrize("env", [dict(GUM_TAIL_NODEDUPE="1"), dict(GUM_TAIL_NODEDUPE="0"),
                                 dict(GUM_TAIL_NODEDUPE="1", GUM_TAIL_SLACK="0")], ids=["nodedupe", "dedupe", "overflow"])
def test_tail_engine_list_modes(env):
    r = subprocess.run([sys.executable, "-c", f"ROOT = {ROOT!r}\n" + CHILD], cwd=ROOT, env=dict(os.environ, **env),
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    assert r.stdout.count("ok ") == 12, r.stdout
    if env.get("GUM_TAIL_NODEDUPE") == "0":
        assert "overflows 0" in r.stdout, r.stdout  # deduplicated lists never exceed V
