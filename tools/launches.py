"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list (per kernel: count, total, max)."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
h = rows[start]
ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
scale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "second": 1e6, "s": 1e6}
tot, seq = {}, []
for r in rows[start + 1:]:
    name = r[ki].split("(")[0].replace("void ", "").replace("gum::", "")[:40]
    us = float(r[vi].replace(",", "")) * scale[r[ui]]
    tot.setdefault(name, []).append(us)
    seq.append((name, us))
grand = sum(sum(v) for v in tot.values())
for k, v in sorted(tot.items(), key=lambda kv: -sum(kv[1])):
    print(f"{k:42s} n={len(v):5d} total={sum(v):10.1f}us share={sum(v) / grand * 100:5.1f}% max={max(v):9.1f}us")
if len(sys.argv) > 2:
    for n, us in seq:
        print(f"  {n:42s} {us:9.1f}us")
