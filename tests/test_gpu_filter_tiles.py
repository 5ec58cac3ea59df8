"""Filter pass 2 over several tiles per CTA (kernels.cu k_filter, multi-tile branch; the fused dense
tile of BFS/SSSP/WCC/PR without the near-far split). At the parity sizes of the other tests every filter
CTA holds at most one tile; here the filter grid is cut to one CTA per SM (GUM_FILTER_CTAS_PER_SM=1, read
once per process, hence the subprocess) so that a 2^20-vertex bitmap spans 512 dense tiles over 148 CTAs
(stride-permuted), and the results must still equal the oracle's."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import sys
sys.path.insert(0, ROOT)
import inputs
from tests.gpu_helpers import check, csr_of
g = inputs.rmat(20, 16, seed=33)
s = inputs.pick_source(g, 33)
csr = csr_of(g)
for alg in ("bfs", "sssp", "wcc", "pr"):
    for P, part in ((1, "seg"), (1, "degree"), (2, "random")):
        check(g, alg, s, csr=csr, num_gpus=P, part=part)
        print("ok", alg, P, part, flush=True)
"""


def test_filter_multi_tile_per_cta():
    env = dict(os.environ, GUM_FILTER_CTAS_PER_SM="1")
    r = subprocess.run([sys.executable, "-c", f"ROOT = {ROOT!r}\n" + CHILD], cwd=ROOT, env=env,
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    assert r.stdout.count("ok ") == 12, r.stdout


def test_filter_stride_coprime_6159_tiles():
    """with 6159 = 3 * 2053 filter tiles the old stride search (2053 -> 2055) shared the factor 3
    with n_tiles, so a third of the tiles were filtered three times and the rest never. V = 6159 * 2048
    gives 6159 sparse-list tiles (WCC iteration 0, 8 entries per thread) and 6159 dense bitmap tiles (BFS
    forced dense); both must equal the oracle."""
    import numpy as np

    import inputs
    from tests.gpu_helpers import check, csr_of

    V = 6159 * 2048
    rng = np.random.default_rng(6159)
    E = 1 << 20
    src = rng.integers(0, V, E, dtype=np.int64).astype(np.uint32)
    dst = rng.integers(0, V, E, dtype=np.int64).astype(np.uint32)
    g = inputs.EdgeList(V, src, dst, None, "stride6159")
    csr = csr_of(g)
    check(g, "wcc", 0, csr=csr)
    s = int(src[0])
    check(g, "bfs", s, csr=csr, force_mode="dense", tail_vertices=0)
    check(g, "bfs", s, csr=csr, force_mode="sparse", tail_vertices=0)


CHILD_TWO_PASS = r"""
import sys
sys.path.insert(0, ROOT)
import inputs
from tests.gpu_helpers import check, csr_of
g = inputs.rmat(16, 16, seed=35)
s = inputs.pick_source(g, 35)
csr = csr_of(g)
for alg in ("bfs", "sssp", "wcc", "pr"):
    for kw in (dict(), dict(num_gpus=3, part="random"), dict(force_mode="sparse", tail_vertices=0),
               dict(force_mode="dense", tail_vertices=0)):
        check(g, alg, s, csr=csr, **kw)
        print("ok", alg, flush=True)
"""


@pytest.mark.parametrize("onepass", ["0", "1"])
def test_filter_one_and_two_pass(onepass):
    """The one-pass filter (default: one packed atomic reserves each tile's queue and edge ranges) and the
    two-pass reduce-then-scan filter (GUM_FILTER_ONEPASS=0, read once per process) give the oracle's results
    for every algorithm, on one and three workers, forced sparse and dense."""
    env = dict(os.environ, GUM_FILTER_ONEPASS=onepass, GUM_FILTER_CTAS_PER_SM="1")
    r = subprocess.run([sys.executable, "-c", f"ROOT = {ROOT!r}\n" + CHILD_TWO_PASS], cwd=ROOT, env=env,
                       capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    assert r.stdout.count("ok ") == 16, r.stdout
