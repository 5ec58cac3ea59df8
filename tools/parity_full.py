#!/usr/bin/env python
"""Full-size parity of the CUDA path against the oracle on the BASELINE configs.

For each config the graph is generated at full size, run through the C ABI in the launch configuration
bench.py times (same partition, tail engine, near-far split), and compared with the oracle:
  C2 BFS    bit-exact depths on `--sources` sampled sources (FIFO BFS)
  C3 SSSP   bit-exact distances from the corner (binary-heap Dijkstra, u64)
  C4 WCC    bit-exact min-id labels (union-find)
  C5 PR     K = 20, d = 0.85: per-vertex rel <= 1e-5 and L1 <= 1e-6 (OpenMP pull power iteration, which is
            bit-identical to the serial oracle_pagerank -- tests/test_oracle.py)
The result of every config is written to profiles/round2/parity_full_<C>.json.

  python tools/parity_full.py --configs C3,C4,C5 [--sources 4] [--out profiles/round2]
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402  (pick_sources and the bench defaults)
import inputs  # noqa: E402
import oracle  # noqa: E402


def ctx_kwargs(config, alg):
    tail = 0 if (alg == "bfs" and config in ("C1", "C2")) else (65536 if config == "C3" else 16384)  # = bench.py
    return dict(fsteal=True, osteal=True, sssp_delta=4096 if config == "C3" else 0, tail_vertices=tail)


def check(config, n_sources=4, part=None):
    import paper_conf_icde_menggltyz23_b200 as gum

    alg = bench.DEFAULT_ALG[config]
    part = part or ("degree" if alg in ("bfs", "pr") else "seg")  # bench.py's layouts
    t0 = time.perf_counter()
    g = inputs.make_config(config, weighted=(alg == "sssp"))
    sources, outdeg = bench.pick_sources(g, int(config[1]), n_sources)
    if config == "C3":
        sources = [0]
    if alg in ("wcc", "pr"):
        sources = sources[:1]
    row_ptr, col, w = gum.build_csr(g.num_vertices, g.src, g.dst, g.w if alg == "sssp" else None)
    t_gen = time.perf_counter() - t0
    rec = {"config": config, "workload": bench.WORKLOADS[config], "alg": alg, "partition": part,
           "ctx": ctx_kwargs(config, alg), "V": g.num_vertices, "E": g.num_edges, "sources": []}
    ctx = gum.Context(**ctx_kwargs(config, alg))
    ctx.load_csr(row_ptr, col, w)
    ctx.partition(part, 1)
    ctx.prepare(alg)
    gpu = {}
    for s in sources:
        st = ctx.run(alg, s)
        gpu[s] = (ctx.result().copy(), st)
    ctx.close()
    del row_ptr, col, w
    ok_all = True
    t_or = time.perf_counter()
    if alg in ("bfs", "sssp"):
        adj = oracle.Adjacency(g.num_vertices, g.src, g.dst, g.w if alg == "sssp" else None)
    for s in sources:
        out, st = gpu[s]
        if alg == "bfs":
            ref = oracle.bfs(adj, s)
        elif alg == "sssp":
            ref = oracle.sssp(adj, s)
        elif alg == "wcc":
            ref = oracle.wcc(g.num_vertices, g.src, g.dst)
        else:
            ref, threads = oracle.pagerank_pull(g.num_vertices, g.src, g.dst, 20, 0.85)
            rec["oracle_threads"] = threads
        if alg == "pr":
            rel = float(np.max(np.abs(out - ref) / ref))
            l1 = float(np.abs(out - ref).sum())
            ok = rel <= 1e-5 and l1 <= 1e-6
            rec["sources"].append({"source": None, "iterations": st.iterations, "max_rel": rel, "l1": l1,
                                   "ok": ok, "mass": float(out.sum())})
        else:
            mism = int((out != ref).sum())
            ok = mism == 0
            rec["sources"].append({"source": int(s), "iterations": st.iterations, "mismatches": mism, "ok": ok,
                                   "reached": int((ref != 0xFFFFFFFF).sum()), "tail_iterations": st.tail_iterations})
        ok_all &= ok
    rec["oracle_s"] = round(time.perf_counter() - t_or, 1)
    rec["setup_s"] = round(t_gen, 1)
    rec["exact"] = bool(ok_all)
    rec["rule"] = "rel<=1e-5, L1<=1e-6 at K=20" if alg == "pr" else "bit-exact"
    return rec


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C3,C4,C5")
    ap.add_argument("--sources", type=int, default=4)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "round2"))
    args = ap.parse_args()
    os.makedirs(args.out, exist_ok=True)
    bad = 0
    for c in args.configs.split(","):
        rec = check(c, args.sources)
        print(json.dumps(rec), flush=True)
        with open(os.path.join(args.out, f"parity_full_{c}.json"), "w") as f:
            json.dump(rec, f, indent=1)
        bad += 0 if rec["exact"] else 1
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
