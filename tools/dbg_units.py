import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import inputs, oracle
from tests.gpu_helpers import gpu_run, csr_of
g = inputs.rmat(13, 16, seed=51, scramble=False)
s = inputs.pick_source(g, 51)
ref = oracle.run("bfs", g, s)
csr = csr_of(g)
for kw in (dict(num_gpus=3, split_units=True), dict(num_gpus=4, part="random", seed=2, split_units=True),
           dict(num_gpus=4, host_loop=True, split_units=True),
           dict(num_gpus=8, osteal_threshold=1 << 30, osteal_edges_per_worker=30000, split_units=True),
           dict(num_gpus=8, osteal_threshold=1 << 30, osteal_edges_per_worker=30000),
           dict(num_gpus=8, osteal_threshold=1 << 30, osteal_edges_per_worker=30000, split_units=True, tail_vertices=0),
           dict(num_gpus=3, split_units=True, tail_vertices=0)):
    bad = []
    for rep in range(int(os.environ.get("REPS", "30"))):
        out, st, _ = gpu_run(g, "bfs", s, csr=csr, **kw)
        m = int((out != ref).sum())
        if m:
            bad.append((m, st.iterations, st.tail_iterations, st.unit_barriers, st.unit_last_iter))
    print(kw, "failures", len(bad), bad[:3], flush=True)
