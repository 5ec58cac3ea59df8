#!/usr/bin/env python
"""One compute-sanitizer case (tools/sanitize.sh): every algorithm on RMAT-12 in one launch mode, checked
against the oracle (so the sanitizer run is also a parity run).

  python tools/sanitize_case.py single|virtual4|split4|mp2[_hl]   (mp2 is started by torchrun; _hl = host loop)
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import inputs  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icde_menggltyz23_b200 as gum  # noqa: E402

mode = sys.argv[1]
host_loop = mode.endswith("_hl")  # the host-driven loop instead of the CUDA-graph loop
mode = mode[:-3] if host_loop else mode
g = inputs.rmat(12, 16, seed=12)
s = inputs.pick_source(g, 12)
row_ptr, col, w = gum.build_csr(g.num_vertices, g.src, g.dst, g.w)
kw = {"single": dict(num_gpus=1), "virtual4": dict(num_gpus=4, chunk_edges=64, tail_vertices=64),
      "split4": dict(num_gpus=4, split_units=True, tail_vertices=64, osteal_threshold=1 << 30,
                     osteal_edges_per_worker=20000), "mp2": dict(tail_vertices=64)}[mode]
if host_loop:
    kw["host_loop"] = True
if mode == "mp2":
    import torch.distributed as dist

    from paper_conf_icde_menggltyz23_b200 import dist as gdist

    dist.init_process_group("gloo")
    ctx = gdist.mp_context(device=0, **kw)
else:
    ctx = gum.Context(**kw)
bad = []
with ctx:
    ctx.load_csr(row_ptr, col, w)
    ctx.partition("random" if mode != "single" else "degree", 3)
    for alg in ("bfs", "sssp", "wcc", "pr", "dpr"):
        ctx.run(alg, s)
        out = ctx.result()
        if alg == "dpr":
            ok = float(np.abs(out - oracle.delta_pagerank(g.num_vertices, g.src, g.dst, 0.85)).sum()) <= 2e-6
        elif alg == "pr":
            ref = oracle.run("pr", g)
            ok = float(np.max(np.abs(out - ref) / ref)) <= 1e-5
        else:
            ok = bool(np.array_equal(out, oracle.run(alg, g, s)))
        if not ok:
            bad.append(alg)
print(f"SANITIZE_CASE {mode}{'_hl' if host_loop else ''} parity_ok={not bad} bad={bad}", flush=True)
