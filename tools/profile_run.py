"""One configurable GUM run for ncu captures (host-loop mode: every kernel is a separate launch).

  python tools/profile_run.py --config C2 --alg bfs --runs 1
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import inputs  # noqa: E402
import paper_conf_icde_menggltyz23_b200 as gum  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--alg", default="bfs")
ap.add_argument("--runs", type=int, default=1)
ap.add_argument("--gpus", type=int, default=1)
ap.add_argument("--host-loop", type=int, default=1)
ap.add_argument("--part", default="seg")
ap.add_argument("--rmat", type=int, default=0, help="instead of --config: RMAT of this scale (EF 16, seed 9)")
ap.add_argument("--noscramble", action="store_true")
ap.add_argument("--grid", type=int, default=0, help="instead of --config: n x n grid (seed 3), source 0")
ap.add_argument("--osteal-threshold", type=int, default=0)
ap.add_argument("--tail", type=int, default=None, help="tail engine threshold (default: bench.py's choice)")
ap.add_argument("--delta", type=int, default=None, help="SSSP near-far split (default: bench.py's, 4096 on C3)")
a = ap.parse_args()
if a.grid:
    g = inputs.grid(a.grid, seed=3)
    s = 0
elif a.rmat:
    g = inputs.rmat(a.rmat, 16, seed=9, scramble=not a.noscramble, weighted=(a.alg == "sssp"))
    s = inputs.pick_source(g, 9)
else:
    g = inputs.make_config(a.config, weighted=(a.alg == "sssp"))
    s = 0 if a.config == "C3" else inputs.pick_source(g, int(a.config[1]))
rp, col, w = gum.build_csr(g.num_vertices, g.src, g.dst, g.w if a.alg == "sssp" else None)
delta = a.delta if a.delta is not None else (4096 if a.config == "C3" and a.alg == "sssp" else 0)
tail = a.tail if a.tail is not None else (0 if a.alg == "bfs" and a.config in ("C1", "C2") and not (a.rmat or a.grid)
                                          else (65536 if a.config == "C3" and not (a.rmat or a.grid) else 16384))
with gum.Context(num_gpus=a.gpus, host_loop=bool(a.host_loop), profile=bool(a.host_loop), sssp_delta=delta,
                 osteal_threshold=a.osteal_threshold, tail_vertices=tail) as ctx:
    ctx.load_csr(rp, col, w)
    ctx.partition(a.part, 1)
    ctx.prepare(a.alg)
    for _ in range(a.runs):
        st = ctx.run(a.alg, s)
    print(st)
    if a.host_loop:
        print(ctx.profile())
