"""Per-kernel device time of one config under several libgum builds (tuning aid; not a bench value).

  python tools/kbench.py --config C2 --alg bfs --runs 8 [--libs a.so,b.so]

For each library: the graph-mode time per run (CUDA events, gum_run_stats.ms) and the profile-mode
per-kernel sums per run (CUDA events around every launch, GUM_CFG_PROFILE). Each library is loaded in a
fresh subprocess (GUM_LIB) so builds never mix.
"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def child(a):
    sys.path.insert(0, ROOT)
    import numpy as np

    import inputs
    import paper_conf_icde_menggltyz23_b200 as gum

    g = inputs.make_config(a.config, weighted=(a.alg == "sssp"))
    seed = int(a.config[1])
    srcs = [0] if a.config == "C3" else [inputs.pick_source(g, seed + i) for i in range(4)]
    rp, col, w = gum.build_csr(g.num_vertices, g.src, g.dst, g.w if a.alg == "sssp" else None)
    kw = json.loads(a.kw)
    out = {}
    with gum.Context(**kw) as ctx:
        ctx.load_csr(rp, col, w)
        ctx.partition(a.part)
        ctx.prepare(a.alg)
        ref = {}
        for s in srcs:
            ctx.run(a.alg, s)
            ref[s] = ctx.result().copy()
        ms = []
        for i in range(a.runs):
            ms.append(ctx.run(a.alg, srcs[i % len(srcs)]).ms)
        out["graph_ms"] = float(np.median(ms))
        out["graph_ms_min"] = float(np.min(ms))
    with gum.Context(profile=True, **kw) as ctx:
        ctx.load_csr(rp, col, w)
        ctx.partition(a.part)
        ctx.prepare(a.alg)
        ctx.run(a.alg, srcs[0])
        acc = {}
        for i in range(a.runs):
            s = srcs[i % len(srcs)]
            ctx.run(a.alg, s)
            ok = np.array_equal(ctx.result(), ref[s]) if a.alg != "pr" else True
            out.setdefault("same_result", True)
            out["same_result"] &= bool(ok)
            for k, v in ctx.profile().items():
                acc[k] = acc.get(k, 0) + v
        out["profile_per_run"] = {k: round(v / a.runs, 4) for k, v in acc.items() if k.endswith("_ms")}
    print("KBENCH " + json.dumps(out), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--alg", default="bfs")
    ap.add_argument("--runs", type=int, default=8)
    ap.add_argument("--libs", default="")
    ap.add_argument("--kw", default="{}")
    ap.add_argument("--part", default="seg")
    ap.add_argument("--child", action="store_true")
    a = ap.parse_args()
    if a.child:
        return child(a)
    libs = [x for x in a.libs.split(",") if x] or [os.path.join(ROOT, "paper_conf_icde_menggltyz23_b200", "libgum.so")]
    for lib in libs:
        env = dict(os.environ, GUM_LIB=os.path.abspath(lib))
        r = subprocess.run([sys.executable, __file__, "--child", "--config", a.config, "--alg", a.alg, "--runs",
                            str(a.runs), "--kw", a.kw, "--part", a.part], env=env, capture_output=True, text=True)
        line = [x for x in r.stdout.splitlines() if x.startswith("KBENCH ")]
        print(os.path.basename(lib), line[0][7:] if line else ("FAILED " + r.stderr[-800:]), flush=True)


if __name__ == "__main__":
    main()
