import sys; sys.path.insert(0, ".")
import numpy as np, inputs, oracle
import paper_conf_icde_menggltyz23_b200 as gum
from tests.gpu_helpers import csr_of
g = inputs.rmat(13, 16, seed=21); s = inputs.pick_source(g, 21); rp, col, w = csr_of(g)
for alg in ("wcc", "sssp", "bfs"):
    ref = oracle.run(alg, g, s)
    for P in (1, 2, 3):
        for tail in (8192, 64):
            bad_res = bad_cons = 0
            with gum.Context(num_gpus=P, tail_vertices=tail) as ctx:
                ctx.load_csr(rp, col, w if alg == "sssp" else None); ctx.partition()
                for rep in range(100):
                    st = ctx.run(alg, s); out = ctx.result()
                    bad_res += not np.array_equal(out, ref)
                    bad_cons += st.edges_expanded != st.edges_frontier
            print(alg, P, tail, "bad results", bad_res, "conservation misses", bad_cons, flush=True)
