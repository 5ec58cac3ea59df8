"""Debug: which (V, graph, alg) combinations break with the filter tile swizzle."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import inputs, oracle
import paper_conf_icde_menggltyz23_b200 as gum

def run(V, E, alg, seed=1, **kw):
    rng = np.random.default_rng(seed)
    src = rng.integers(0, V, E, dtype=np.int64).astype(np.uint32)
    dst = rng.integers(0, V, E, dtype=np.int64).astype(np.uint32)
    g = inputs.EdgeList(V, src, dst, None, "x")
    rp, col, _ = gum.build_csr(V, src, dst, None)
    s = int(src[0])
    try:
        with gum.Context(**kw) as ctx:
            ctx.load_csr(rp, col)
            ctx.partition("seg", 0)
            st = ctx.run(alg, s)
            out = ctx.result()
        ref = oracle.run(alg, g, s)
        return f"mism={int((out != ref).sum())} iters={st.iterations}"
    except Exception as e:
        return f"EXC {str(e)[:120]}"

cases = [(6159 * 2048, 1 << 20, "wcc", {}), (6160 * 2048, 1 << 20, "wcc", {}), (6159 * 2048, 1 << 20, "wcc", {"tail_vertices": 0}),
         (6159 * 2048, 1 << 20, "bfs", {"force_mode": "dense", "tail_vertices": 0}), (8192 * 2048, 1 << 20, "wcc", {}),
         (6159 * 2048, 1 << 23, "wcc", {}), (4096 * 2048, 1 << 20, "wcc", {}), (3000 * 2048, 1 << 20, "wcc", {})]
if len(sys.argv) > 1:
    V, E, alg, kw = cases[int(sys.argv[1])]
    print(V // 2048, E, alg, kw, run(V, E, alg, **kw), flush=True)
else:
    import subprocess
    for i in range(len(cases)):
        subprocess.run([sys.executable, __file__, str(i)])
