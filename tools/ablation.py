"""FSteal / OSteal ablations from the device-side per-iteration trace.

FSteal: per iteration, worker w's advance busy window [t_start[w], t_end[w]] (%globaltimer, min start /
max end over its CTAs); spread = slowest / fastest worker, starvation = sum_w (max busy - busy_w).
Run with stealing on vs off on a statically skewed partition (unscrambled RMAT, seg ranges).

OSteal: SSSP on a high-diameter grid; total time and the time spent after the active vertex count
drops below the OSteal threshold ("long tail"), OSteal on vs off.

  python tools/ablation.py --fsteal --scale 22 --workers 8 [--split]
  python tools/ablation.py --osteal --grid 2048 --workers 8 [--split]

NEXT-1: cross-fragment traffic with and without outer-vertex mirrors and the hub cache, per
algorithm on RMAT with a random partition over 8 workers: remote atomics issued (each one crosses NVLink when
the workers are GPUs), updates absorbed by the mirrors, PR mirror bytes pulled per run, stolen edges read
from a local hub copy. Outputs must be identical (PR: within the parity tolerance).

  python tools/ablation.py --next1 --scale 20 --workers 8

NEXT-2 / Table IV: FSteal off vs the steal queue ("peek-and-grab") vs the planned
estimate-and-reassign FSteal (Eq. (1) + Alg. 1), and OSteal off vs the cost model (Alg. 2 / Eq. (4) with online
p), on 8 virtual workers: run time, time saved against "off", and the overhead -- the extra time of the
control kernel (gating, planning, owner decisions; CUDA events per launch in a profile pass) -- with the
paper's ratio saved / overhead.

  python tools/ablation.py --table4 --scale 22 --grid 2048 --workers 8
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import inputs  # noqa: E402
import paper_conf_icde_menggltyz23_b200 as gum  # noqa: E402


TAIL = None  # --tail: tail engine threshold override


def run(csr, alg, src, reps=3, **kw):
    rp, col, w = csr
    if TAIL is not None:
        kw.setdefault("tail_vertices", TAIL)
    with gum.Context(trace=True, **kw) as ctx:
        ctx.load_csr(rp, col, w if alg == "sssp" else None)
        ctx.partition("seg")
        ctx.run(alg, src)  # warm
        best = None
        for _ in range(reps):
            st = ctx.run(alg, src)
            tr = ctx.trace()
            if best is None or st.ms < best[0].ms:
                best = (st, tr)
        out = ctx.result()
    return best[0], best[1], out


def spread_stats(tr, P):
    rows = []
    for k, r in enumerate(tr):
        busy = [(r["t_end"][w] - r["t_start"][w]) / 1e3 if r["t_end"][w] else 0.0 for w in range(P)]
        active = [b for b in busy if b > 0]
        if not active:
            continue
        mx, mn = max(active), min(active)
        dur = (max(r["t_end"][w] for w in range(P) if r["t_end"][w]) -
               min(r["t_start"][w] for w in range(P) if r["t_end"][w])) / 1e3
        rows.append(dict(iter=k, frontier_edges=r["frontier_edges"], steal_ok=r["steal_ok"], owners=r["owners"],
                         busy_us=[round(b, 1) for b in busy], spread=round(mx / mn, 3) if mn > 0 else None,
                         starvation_us=round(sum(mx - b for b in busy), 1), advance_us=round(dur, 1),
                         stolen_edges=sum(r["edges_stolen"])))
    return rows


def fsteal(args):
    g = inputs.rmat(args.scale, 16, seed=9, scramble=False, weighted=False)
    src = inputs.pick_source(g, 9)
    csr = gum.build_csr(g.num_vertices, g.src, g.dst)
    res = {}
    for on in (True, False):
        st, tr, out = run(csr, "bfs", src, num_gpus=args.workers, fsteal=on, split_units=args.split,
                          chunk_edges=args.chunk)
        rows = spread_stats(tr, args.workers)
        big = [r for r in rows if r["frontier_edges"] >= 0.05 * max(x["frontier_edges"] for x in rows)]
        res["on" if on else "off"] = dict(
            run_ms=st.ms, iterations=st.iterations, chunks_stolen=st.chunks_stolen, edges_stolen=st.edges_stolen,
            advance_us_total=round(sum(r["advance_us"] for r in rows), 1),
            max_spread_big_iters=max((r["spread"] or 1) for r in big),
            starvation_us_total=round(sum(r["starvation_us"] for r in rows), 1), per_iteration=rows)
        res.setdefault("outputs", []).append(out)
    same = bool(np.array_equal(res["outputs"][0], res["outputs"][1]))
    del res["outputs"]
    res["identical_outputs"] = same
    res["workload"] = (f"BFS RMAT-{args.scale} EF16 unscrambled (hubs at low ids), seg partition, "
                       f"{args.workers} {'split-unit' if args.split else 'virtual'} workers on 1 B200, "
                       f"chunk {args.chunk} edges, source {src}")
    return res


def osteal(args):
    g = inputs.grid(args.grid, seed=3)
    csr = gum.build_csr(g.num_vertices, g.src, g.dst, g.w)
    res = {}
    thr = args.threshold
    for on in (True, False):
        st, tr, out = run(csr, "sssp", 0, reps=2, num_gpus=args.workers, osteal=on, osteal_threshold=thr,
                          split_units=args.split, sssp_delta=args.delta)
        rows = spread_stats(tr, args.workers)
        tail = [r for r in rows if tr[r["iter"]]["frontier_vertices"] < thr]
        res["on" if on else "off"] = dict(run_ms=st.ms, iterations=st.iterations, final_owners=st.final_owners,
                                          osteal_iteration=st.osteal_iteration,
                                          tail_iterations=len(tail),
                                          tail_advance_us=round(sum(r["advance_us"] for r in tail), 1))
        res.setdefault("outputs", []).append(out)
    res["identical_outputs"] = bool(np.array_equal(res["outputs"][0], res["outputs"][1]))
    del res["outputs"]
    res["workload"] = (f"SSSP on a {args.grid}x{args.grid} grid (w in [1,255]), source 0, {args.workers} "
                       f"{'split-unit' if args.split else 'virtual'} workers on 1 B200, OSteal threshold {thr} "
                       f"active vertices; near-far delta {args.delta}; OSteal on includes the m'=1 tail engine "
                       f"(on unit 0 across every fragment; with --split the other units park in their graphs)")
    return res


def next1(args):
    g = inputs.rmat(args.scale, 16, seed=2)
    src = inputs.pick_source(g, 2)
    csr = gum.build_csr(g.num_vertices, g.src, g.dst, g.w)
    res = {}
    for alg in ("bfs", "sssp", "wcc", "pr"):
        rows = {}
        outs = []
        for name, kw in (("plain", {}), ("mirrors", dict(mirrors=True)),
                         ("mirrors+hub", dict(mirrors=True, hub_cache=True, hub_degree=args.hub_degree))):
            rp, col, w = csr
            with gum.Context(num_gpus=args.workers, chunk_edges=args.chunk, **kw) as ctx:
                ctx.load_csr(rp, col, w if alg == "sssp" else None)
                ctx.partition("random", 1)
                ctx.run(alg, src)
                st = min((ctx.run(alg, src) for _ in range(3)), key=lambda t: t.ms)
                outs.append(ctx.result())
            op = 8 if alg == "pr" else 4
            rows[name] = dict(run_ms=round(st.ms, 3), iterations=st.iterations, remote_atomics=st.remote_updates,
                              remote_atomic_bytes=st.remote_updates * op, absorbed_by_mirror=st.remote_filtered,
                              mirror_flush_bytes=st.mirror_flush_bytes, edges_stolen=st.edges_stolen,
                              stolen_edges_from_hub_copy=st.hub_cached_edges)
        if alg == "pr":
            ok = all(float(np.abs(o - outs[0]).sum()) <= 1e-6 for o in outs)
        else:
            ok = all(np.array_equal(o, outs[0]) for o in outs)
        rows["identical_outputs"] = bool(ok)
        res[alg] = rows
    res["workload"] = (f"RMAT scale {args.scale} EF16 (seed 2), random partition over {args.workers} virtual workers "
                       f"on 1 B200, chunk {args.chunk} edges, hub t4 = {args.hub_degree}; remote atomic bytes = "
                       f"count x 4 B (8 B for PR's fp64 adds); on one GPU every access stays in HBM, so the times "
                       f"are not NVLink times -- the counts are the cross-GPU traffic the same run issues on N GPUs")
    return res


def profile_ms(csr, alg, src, reps=3, **kw):
    """Per-kernel device time per run (profile pass: host loop, CUDA events around every launch)."""
    rp, col, w = csr
    with gum.Context(profile=True, **kw) as ctx:
        ctx.load_csr(rp, col, w if alg == "sssp" else None)
        ctx.partition("seg")
        ctx.run(alg, src)
        acc = {}
        for _ in range(reps):
            ctx.run(alg, src)
            for k, v in ctx.profile().items():
                if k.endswith("_ms"):
                    acc[k] = acc.get(k, 0.0) + v / reps
    return acc


def table4(args):
    res = {}
    g = inputs.rmat(args.scale, 16, seed=9, scramble=False, weighted=False)
    src = inputs.pick_source(g, 9)
    csr = gum.build_csr(g.num_vertices, g.src, g.dst)
    modes = (("off", dict(fsteal=False)), ("queue", dict(fsteal=True)), ("planned", dict(fsteal="planned")))
    fs, outs = {}, []
    for name, kw in modes:
        st, tr, out = run(csr, "bfs", src, num_gpus=args.workers, chunk_edges=args.chunk, **kw)
        rows = spread_stats(tr, args.workers)
        big = [r for r in rows if r["frontier_edges"] >= 0.05 * max(x["frontier_edges"] for x in rows)]
        prof = profile_ms(csr, "bfs", src, num_gpus=args.workers, chunk_edges=args.chunk, **kw)
        fs[name] = dict(run_ms=round(st.ms, 4), advance_us_total=round(sum(r["advance_us"] for r in rows), 1),
                        max_spread_big_iters=max((r["spread"] or 1) for r in big),
                        starvation_us_total=round(sum(r["starvation_us"] for r in rows), 1),
                        chunks_stolen=st.chunks_stolen, edges_stolen=st.edges_stolen,
                        control_ms=round(prof.get("control_ms", 0.0), 4), advance_ms=round(prof.get("advance_ms", 0.0), 4))
        outs.append(out)
    for name in ("queue", "planned"):
        saved = fs["off"]["run_ms"] - fs[name]["run_ms"]
        over = max(fs[name]["control_ms"] - fs["off"]["control_ms"], 0.0)
        fs[name].update(saved_ms=round(saved, 4), overhead_ms=round(over, 4),
                        ratio=round(saved / over, 1) if over > 0 else None)
    fs["identical_outputs"] = all(np.array_equal(o, outs[0]) for o in outs)
    fs["workload"] = (f"BFS RMAT-{args.scale} EF16 unscrambled (hubs at low ids: a statically skewed seg partition), "
                      f"{args.workers} virtual workers on 1 B200, chunk {args.chunk}")
    res["fsteal"] = fs
    gg = inputs.grid(args.grid, seed=3)
    gcsr = gum.build_csr(gg.num_vertices, gg.src, gg.dst, gg.w)
    os_, outs = {}, []
    for name, kw in (("off", dict(osteal=False)), ("cost", dict(osteal="cost", osteal_sync_edges=0.0))):
        st, tr, out = run(gcsr, "sssp", 0, reps=2, num_gpus=args.workers, sssp_delta=args.delta, tail_vertices=0, **kw)
        prof = profile_ms(gcsr, "sssp", 0, reps=1, num_gpus=args.workers, sssp_delta=args.delta, tail_vertices=0, **kw)
        os_[name] = dict(run_ms=round(st.ms, 3), iterations=st.iterations, final_owners=st.final_owners,
                         osteal_iteration=st.osteal_iteration, osteal_p=st.osteal_p, p_samples=st.osteal_p_samples,
                         control_ms=round(prof.get("control_ms", 0.0), 3), advance_ms=round(prof.get("advance_ms", 0.0), 3))
        outs.append(out)
    saved = os_["off"]["run_ms"] - os_["cost"]["run_ms"]
    over = max(os_["cost"]["control_ms"] - os_["off"]["control_ms"], 0.0)
    os_["cost"].update(saved_ms=round(saved, 3), overhead_ms=round(over, 3), ratio=round(saved / over, 1) if over > 0 else None)
    os_["identical_outputs"] = bool(np.array_equal(outs[0], outs[1]))
    os_["workload"] = (f"SSSP {args.grid}x{args.grid} grid, near-far delta {args.delta}, {args.workers} virtual workers on "
                       f"1 B200, tail engine off (OSteal's owner shrink alone). On one GPU the evicted workers' CTAs "
                       f"simply go idle: the sync cost OSteal removes across GPUs (barriers, launches per GPU) does "
                       f"not exist here, so 'saved' is not the multi-GPU effect")
    res["osteal"] = os_
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--fsteal", action="store_true")
    ap.add_argument("--osteal", action="store_true")
    ap.add_argument("--scale", type=int, default=22)
    ap.add_argument("--grid", type=int, default=2048)
    ap.add_argument("--workers", type=int, default=8)
    ap.add_argument("--chunk", type=int, default=2048)
    ap.add_argument("--threshold", type=int, default=4096)
    ap.add_argument("--delta", type=int, default=0, help="SSSP near-far split (0 = plain frontier)")
    ap.add_argument("--split", action="store_true")
    ap.add_argument("--next1", action="store_true")
    ap.add_argument("--tail", type=int, default=None, help="tail engine threshold (default: the library's)")
    ap.add_argument("--hub-degree", type=int, default=64)
    ap.add_argument("--table4", action="store_true")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    global TAIL
    TAIL = args.tail
    out = {}
    if args.fsteal:
        out["fsteal"] = fsteal(args)
        f = out["fsteal"]
        print(f"FSteal on : {f['on']['run_ms']:.3f} ms, advance {f['on']['advance_us_total']} us, "
              f"max spread {f['on']['max_spread_big_iters']}, starvation {f['on']['starvation_us_total']} us, "
              f"stolen chunks {f['on']['chunks_stolen']}")
        print(f"FSteal off: {f['off']['run_ms']:.3f} ms, advance {f['off']['advance_us_total']} us, "
              f"max spread {f['off']['max_spread_big_iters']}, starvation {f['off']['starvation_us_total']} us")
    if args.osteal:
        out["osteal"] = osteal(args)
        o = out["osteal"]
        for k in ("on", "off"):
            print(f"OSteal {k}: {o[k]['run_ms']:.2f} ms, {o[k]['iterations']} iterations, owners {o[k]['final_owners']}, "
                  f"tail iterations {o[k]['tail_iterations']}, tail advance {o[k]['tail_advance_us']} us")
    if args.next1:
        out["next1"] = next1(args)
        for alg, rows in out["next1"].items():
            if alg == "workload":
                continue
            for k, r in rows.items():
                if isinstance(r, dict):
                    print(f"{alg:5s} {k:12s} {r['run_ms']:9.3f} ms  remote atomics {r['remote_atomics']:>12d}  "
                          f"absorbed {r['absorbed_by_mirror']:>12d}  flush {r['mirror_flush_bytes']:>12d} B  "
                          f"hub-copy edges {r['stolen_edges_from_hub_copy']}")
            print(f"{alg:5s} identical outputs: {rows['identical_outputs']}")
    if args.table4:
        out["table4"] = table4(args)
        t = out["table4"]
        for k in ("off", "queue", "planned"):
            r = t["fsteal"][k]
            print(f"FSteal {k:8s} {r['run_ms']:8.3f} ms  spread {r['max_spread_big_iters']}  starvation "
                  f"{r['starvation_us_total']} us  control {r['control_ms']} ms  saved {r.get('saved_ms')}  "
                  f"overhead {r.get('overhead_ms')}  ratio {r.get('ratio')}")
        for k in ("off", "cost"):
            r = t["osteal"][k]
            print(f"OSteal {k:5s} {r['run_ms']:8.3f} ms  owners {r['final_owners']}  control {r['control_ms']} ms  "
                  f"p {r['osteal_p']:.0f} ({r['p_samples']})  saved {r.get('saved_ms')}  overhead {r.get('overhead_ms')}  "
                  f"ratio {r.get('ratio')}")
    if args.out:
        json.dump(out, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
