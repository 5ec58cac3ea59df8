import sys, time; sys.path.insert(0, ".")
import numpy as np, inputs, oracle
import paper_conf_icde_menggltyz23_b200 as gum
from tests.gpu_helpers import csr_of
g = inputs.rmat(13, 16, seed=51); s = inputs.pick_source(g, 51); rp, col, w = csr_of(g)
ref = oracle.run("sssp", g, s)
for tail in (0, 8192):
    for delta in (600, 37, 1):
        with gum.Context(sssp_delta=delta, tail_vertices=tail, host_loop=True, max_iterations=200000) as ctx:
            ctx.load_csr(rp, col, w); ctx.partition()
            t = time.time(); st = ctx.run("sssp", s); out = ctx.result()
            print(tail, delta, np.array_equal(out, ref), st.iterations, st.tail_iterations, st.bodies, round(time.time() - t, 3), flush=True)
