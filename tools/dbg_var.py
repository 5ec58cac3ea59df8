import sys, os; sys.path.insert(0, ".")
import numpy as np, inputs, oracle
import paper_conf_icde_menggltyz23_b200 as gum
g = inputs.make_config("C2", weighted=False)
srcs = [inputs.pick_source(g, 2)]
rp, col, w = gum.build_csr(g.num_vertices, g.src, g.dst)
for chunk in (1024, 512, 2048):
    with gum.Context(chunk_edges=chunk) as ctx:
        ctx.load_csr(rp, col); ctx.partition(); ctx.run("bfs", srcs[0])
        ms = min(ctx.run("bfs", srcs[0]).ms for _ in range(5))
        print(os.environ.get("GUM_LIB", "default"), "chunk", chunk, "ms", round(ms, 3), flush=True)
