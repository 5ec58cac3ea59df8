import sys; sys.path.insert(0, ".")
import numpy as np, inputs
import paper_conf_icde_menggltyz23_b200 as gum
from tests.gpu_helpers import csr_of
g = inputs.from_pairs(3, [(0, 1), (1, 2)], [0xFFFFFFF0, 0x20])
rp, col, w = csr_of(g)
for kw in (dict(tail_vertices=0), dict()):
    with gum.Context(**kw) as ctx:
        ctx.load_csr(rp, col, w); ctx.partition()
        print(kw, "sssp", flush=True)
        try:
            ctx.run("sssp", 0)
        except gum.GumError as e:
            print("  sssp err", e.status, flush=True)
        print("  bfs", flush=True)
        st = ctx.run("bfs", 0); print("  bfs ok", ctx.result().tolist(), st.iterations, st.tail_iterations, flush=True)
