import sys, time; sys.path.insert(0, ".")
import numpy as np, inputs, oracle
import paper_conf_icde_menggltyz23_b200 as gum
from tests.gpu_helpers import csr_of
for scale in (13, 18, 20):
    g = inputs.rmat(scale, 16, seed=scale, weighted=False); s = inputs.pick_source(g, scale); rp, col, w = csr_of(g)
    ref = oracle.run("bfs", g, s)
    for pbl in (17, 0):
        with gum.Context(pb_block_log2=pbl) as ctx:
            ctx.load_csr(rp, col); ctx.partition()
            bad = 0
            for rep in range(20):
                st = ctx.run("bfs", s); bad += not np.array_equal(ctx.result(), ref)
            print(scale, pbl, "bad", bad, "ms", round(st.ms, 3), "iters", st.iterations, st.edges_expanded == st.edges_frontier, flush=True)
