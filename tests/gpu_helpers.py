"""Shared helpers of the -m gpu parity tests: run the CUDA path through the C ABI and the oracle on
the same seeded edge list."""
import numpy as np

import oracle
import paper_conf_icde_menggltyz23_b200 as gum


def csr_of(g):
    return gum.build_csr(g.num_vertices, g.src, g.dst, g.w)


def gpu_run(g, alg, source=0, csr=None, part="seg", seed=0, **ctx_kw):
    row_ptr, col, w = csr if csr is not None else csr_of(g)
    with gum.Context(**ctx_kw) as ctx:
        ctx.load_csr(row_ptr, col, w if alg == "sssp" else None)
        ctx.partition(part, seed)
        st = ctx.run(alg, source)
        out = ctx.result()
        tr = ctx.trace() if ctx_kw.get("trace") else None
    return out, st, tr


def assert_pr_close(x, ref):
    rel = np.abs(x - ref) / ref
    assert rel.max() <= 1e-5, f"max rel err {rel.max()}"
    assert np.abs(x - ref).sum() <= 1e-6, f"L1 {np.abs(x - ref).sum()}"


def check(g, alg, source=0, csr=None, ref=None, **kw):
    out, st, tr = gpu_run(g, alg, source, csr=csr, **kw)
    if ref is None:
        ref = oracle.run(alg, g, source)
    if alg == "pr":
        assert_pr_close(out, ref)
    else:
        bad = np.nonzero(out != ref)[0]
        assert bad.size == 0, f"{alg}: {bad.size} mismatches, first {bad[:5]} gpu={out[bad[:5]]} ora={ref[bad[:5]]}"
    # conservation: every frontier edge expanded exactly once
    assert st.edges_expanded == st.edges_frontier, (st.edges_expanded, st.edges_frontier)
    return out, st, tr
