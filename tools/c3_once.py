import sys; sys.path.insert(0, ".")
import inputs, paper_conf_icde_menggltyz23_b200 as gum
g = inputs.grid(8192, seed=3); rp, col, w = gum.build_csr(g.num_vertices, g.src, g.dst, g.w)
with gum.Context(sssp_delta=4096) as c:
    c.load_csr(rp, col, w); c.partition(); print(c.run("sssp", 0))
