"""Per-iteration timeline of one config in graph mode (tuning aid; not a bench value).

  python tools/iter_trace.py --config C2 --alg bfs --part degree [--runs 3] [--kw '{...}']

Per BSP iteration: frontier vertices and edges, the advance window (first CTA start to last CTA end,
%globaltimer, gum_trace), and the gap from this advance's end to the next advance's start (filter + control
of the next iteration + launch gaps). Median over runs of the same source.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import inputs  # noqa: E402
import paper_conf_icde_menggltyz23_b200 as gum  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--alg", default="bfs")
ap.add_argument("--part", default="degree")
ap.add_argument("--runs", type=int, default=3)
ap.add_argument("--kw", default="{}")
a = ap.parse_args()
g = inputs.make_config(a.config, weighted=(a.alg == "sssp"))
s = 0 if a.config == "C3" else inputs.pick_source(g, int(a.config[1]))
rp, col, w = gum.build_csr(g.num_vertices, g.src, g.dst, g.w if a.alg == "sssp" else None)
kw = dict(tail_vertices=0 if a.alg == "bfs" else 16384)
kw.update(json.loads(a.kw))
with gum.Context(trace=True, **kw) as ctx:
    ctx.load_csr(rp, col, w)
    ctx.partition(a.part, 1)
    ctx.prepare(a.alg)
    ctx.run(a.alg, s)
    rows, ms = [], []
    for _ in range(a.runs):
        st = ctx.run(a.alg, s)
        ms.append(st.ms)
        tr = ctx.trace()
        rows.append([(r["frontier_vertices"], r["frontier_edges"], r["t_start"][0], r["t_end"][0]) for r in tr])
print(f"run ms (graph): median {np.median(ms):.4f}  min {np.min(ms):.4f}  iterations {len(rows[0])}")
n = len(rows[0])
print(f"{'it':>3} {'front_v':>10} {'front_e':>11} {'adv_us':>8} {'gap_us':>8} {'GE/s':>7}")
tot_adv = tot_gap = 0.0
for i in range(n):
    adv = np.median([(r[i][3] - r[i][2]) / 1e3 for r in rows if i < len(r)])
    gap = np.median([(r[i + 1][2] - r[i][3]) / 1e3 for r in rows if i + 1 < len(r)]) if i + 1 < n else 0.0
    fv, fe = rows[0][i][0], rows[0][i][1]
    tot_adv += adv
    tot_gap += gap
    print(f"{i:>3} {fv:>10} {fe:>11} {adv:>8.1f} {gap:>8.1f} {fe / adv / 1e3 if adv > 0 else 0:>7.1f}")
print(f"sum advance windows {tot_adv:.1f} us, sum gaps {tot_gap:.1f} us")
