import sys; sys.path.insert(0, ".")
import inputs, paper_conf_icde_menggltyz23_b200 as gum
d = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
g = inputs.grid(8192, seed=3); rp, col, w = gum.build_csr(g.num_vertices, g.src, g.dst, g.w)
with gum.Context(sssp_delta=d, profile=True) as c:
    c.load_csr(rp, col, w); c.partition(); st = c.run("sssp", 0)
    print(st); print(c.profile())
