"""C3 (8192^2 grid SSSP) time-to-converge: plain BSP frontier vs near-far deltas, tail engine on/off."""
import sys; sys.path.insert(0, ".")
import json, inputs, paper_conf_icde_menggltyz23_b200 as gum
g = inputs.grid(8192, seed=3); rp, col, w = gum.build_csr(g.num_vertices, g.src, g.dst, g.w)
res = []
for delta in [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "0,1024,4096").split(",")]:
    for tail in (0, 8192):
        with gum.Context(sssp_delta=delta, tail_vertices=tail) as c:
            c.load_csr(rp, col, w); c.partition(); c.run("sssp", 0)
            st = min((c.run("sssp", 0) for _ in range(2)), key=lambda s: s.ms)
            r = dict(delta=delta, tail=tail, ms=round(st.ms, 1), iterations=st.iterations, tail_iterations=st.tail_iterations,
                     bodies=st.bodies, edges_expanded=st.edges_expanded)
            print(json.dumps(r), flush=True); res.append(r)
