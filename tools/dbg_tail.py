import os, sys, subprocess
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if len(sys.argv) > 1:
    import inputs
    from tests.gpu_helpers import gpu_run
    import paper_conf_icde_menggltyz23_b200 as gum
    g = inputs.grid(int(sys.argv[1]), seed=3)
    csr = gum.build_csr(g.num_vertices, g.src, g.dst, g.w)
    for d in (4096, 1024):
        out, st, _ = gpu_run(g, "sssp", 0, csr=csr, sssp_delta=d, tail_vertices=16384)
        out2, st2, _ = gpu_run(g, "sssp", 0, csr=csr, sssp_delta=d, tail_vertices=16384)
        print(os.environ.get("GUM_TAIL_LOCAL"), "delta", d, "iters", st2.iterations, "tail", st2.tail_iterations, "ms", round(st2.ms, 2),
              "edges", st2.edges_expanded, "tailv", st2.tail_vertices, flush=True)
else:
    for L in ("0", "1", "3", "8"):
        subprocess.run([sys.executable, __file__, "4096"], env=dict(os.environ, GUM_TAIL_LOCAL=L))
