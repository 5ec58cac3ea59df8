"""Stall samples per CUDA source line of an ncu report (needs -lineinfo + --import-source on)."""
import csv
import io
import subprocess
import sys

out = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source=cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = next(i for i, r in enumerate(rows) if r and r[0] == "Line No")
h = rows[hdr]
si = h.index("Warp Stall Sampling (All Samples)")
cur, tot, per = None, 0, {}
for r in rows[hdr + 1:]:
    if len(r) <= si:
        continue
    if r[0]:
        cur = (r[0], r[1].strip()[:100])
        continue
    try:
        v = float(r[si])
    except ValueError:
        continue
    per[cur] = per.get(cur, 0) + v
    tot += v
for (ln, src), v in sorted(per.items(), key=lambda kv: -kv[1])[: int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    print(f"{v / tot * 100:5.1f}%  L{ln:>5}  {src}")
