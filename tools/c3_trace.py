"""C3 iteration profile: frontier sizes per BSP iteration (trace) for the near-far SSSP run."""
import sys; sys.path.insert(0, ".")
import numpy as np, inputs, paper_conf_icde_menggltyz23_b200 as gum
d = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
g = inputs.grid(8192, seed=3); rp, col, w = gum.build_csr(g.num_vertices, g.src, g.dst, g.w)
with gum.Context(sssp_delta=d, trace=True) as c:
    c.load_csr(rp, col, w); c.partition(); st = c.run("sssp", 0); tr = c.trace()
print(st)
fv = np.array([r["frontier_vertices"] for r in tr]); fe = np.array([r["frontier_edges"] for r in tr])
print("iterations", len(fv), "frontier vertices: pct", np.percentile(fv, [5, 25, 50, 75, 95, 99]).tolist(), "max", fv.max())
for lo, hi in [(0, 1), (1, 8192), (8192, 32768), (32768, 131072), (131072, 1 << 40)]:
    m = (fv >= lo) & (fv < hi)
    print(f"  [{lo},{hi}): {m.sum()} iterations, {fv[m].sum()} vertices")
