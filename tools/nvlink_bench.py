#!/usr/bin/env python
"""Link micro-benchmark (§III-B: the bandwidth B_ij "can be evaluated via micro benchmark";
SURVEY.md §8(d) "NVLink GB/s"): for every ordered device pair (i executes, memory on j) -- and i = j for local
HBM -- stream-read and stream-write GB/s, random 4-byte atomic rate and dependent-load latency
(tools/linkbench/liblinkbench.so). From them it derives the FSteal remote-edge cost of the planned FSteal,
c_ij = B_ii / B_ij (P:101-108 with the learned term g left out, reading #11), i.e. the value to pass
as gum_config.fsteal_remote_cost.

  python tools/nvlink_bench.py [--bytes 1073741824] [--out profiles/round2/nvlink_bench.json]

On a one-GPU box only the local row is measured and the peer entries are reported as unavailable.
"""
import argparse
import ctypes
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "tools", "linkbench", "liblinkbench.so")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--bytes", type=int, default=1 << 30)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--atomics", type=int, default=1 << 28)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    lib = ctypes.CDLL(LIB)
    d = ctypes.c_double
    lib.lb_stream_bw.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_ulonglong, ctypes.c_int, ctypes.c_int, ctypes.POINTER(d)]
    lib.lb_atomic_rate.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_ulonglong, ctypes.POINTER(d)]
    lib.lb_latency.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_uint, ctypes.POINTER(d)]
    n = lib.lb_device_count()
    if n < 1:
        print(json.dumps({"error": "no CUDA device"}))
        sys.exit(1)
    res = {"devices": n, "pairs": []}
    for i in range(n):
        for j in range(n):
            r, w, at, lat = d(), d(), d(), d()
            st = [lib.lb_stream_bw(i, j, a.bytes, a.reps, 1, ctypes.byref(r)),
                  lib.lb_stream_bw(i, j, a.bytes, a.reps, 0, ctypes.byref(w)),
                  lib.lb_atomic_rate(i, j, a.atomics, ctypes.byref(at)), lib.lb_latency(i, j, 200000, ctypes.byref(lat))]
            rec = {"exec": i, "mem": j, "link": "local HBM" if i == j else "peer (NVLink/NVSwitch)"}
            if any(st):
                rec["error"] = f"status {st} (no peer access?)"
            else:
                rec.update(read_gbs=round(r.value, 1), write_gbs=round(w.value, 1), atomic_gops=round(at.value, 2),
                           latency_ns=round(lat.value, 1))
            res["pairs"].append(rec)
            print(json.dumps(rec), flush=True)
    loc = {p["exec"]: p for p in res["pairs"] if p["exec"] == p["mem"] and "read_gbs" in p}
    costs = {}
    for p in res["pairs"]:
        if p["exec"] != p["mem"] and "read_gbs" in p and p["exec"] in loc:
            costs[f"{p['exec']}->{p['mem']}"] = round(loc[p["exec"]]["read_gbs"] / p["read_gbs"], 2)
    res["fsteal_remote_cost"] = costs or None
    if costs:
        res["fsteal_remote_cost_mean"] = round(sum(costs.values()) / len(costs), 2)
    if n == 1:
        res["note"] = "one GPU: peer links not measurable on this box (local HBM row only)"
    print(json.dumps({k: v for k, v in res.items() if k != "pairs"}), flush=True)
    if a.out:
        os.makedirs(os.path.dirname(a.out), exist_ok=True)
        json.dump(res, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
