import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import inputs, oracle
from tests.gpu_helpers import gpu_run, csr_of
g = inputs.rmat(16, 16, seed=71, scramble=False)
s = inputs.pick_source(g, 71)
csr = csr_of(g)
out, st, tr = gpu_run(g, "bfs", s, csr=csr, fsteal="planned", trace=True, num_gpus=4, tail_vertices=0, chunk_edges=256)
for r in tr:
    print(r["frontier_edges"], r["steal_ok"], r["owners"], [a + b for a, b in zip(r["edges_own"], r["edges_stolen"])], r["edges_stolen"])
