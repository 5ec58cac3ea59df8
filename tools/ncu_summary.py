"""Summarise an ncu --set full report: key metrics + top stall reasons (SASS source page)."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem", "launch__grid_size",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
        "lts__t_requests_srcunit_tex_op_red.sum", "lts__t_requests_srcunit_tex_op_atom.sum",
        "sm__cycles_elapsed.avg.per_second"]
import os

# NCU_IMPORT_ARGS: extra import filters, e.g. "--launch-skip 7 --launch-count 1" (one kernel of a multi-kernel report)
FILT = os.environ.get("NCU_IMPORT_ARGS", "").split()
raw = subprocess.run(["ncu", "-i", rep] + FILT + ["--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, units = rows[0], rows[1]
for r in rows[2:]:
    print("kernel:", r[h.index("Kernel Name")][:80] if "Kernel Name" in h else "")
    for k in KEYS:
        if k in h:
            i = h.index(k)
            print(f"  {k:62s} {r[i]:>18s} {units[i]}")
src = subprocess.run(["ncu", "-i", rep] + FILT + ["--page", "source", "--csv", "--print-source=sass"], capture_output=True,
                     text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
col = "Warp Stall Sampling (All Samples)"
hi = next((i for i, r in enumerate(rows) if col in r), None)  # (the header row; one per kernel in the report)


def num(x):
    try:
        return float(x)
    except ValueError:
        return 0.0


if hi is not None:
    h = rows[hi]
    nxt = next((i for i in range(hi + 1, len(rows)) if col in rows[i]), len(rows))  # (first kernel only)
    data = [r for r in rows[hi + 1:nxt] if len(r) == len(h) and col not in r]
    ix = {n: i for i, n in enumerate(h)}
    tot = sum(num(r[ix[col]]) for r in data) or 1
    stalls = [n for n in h if n.startswith("stall_") and "Not Issued" not in n]
    agg = sorted(((sum(num(r[ix[n]]) for r in data) / tot * 100, n) for n in stalls), reverse=True)[:8]
    print("  stall reasons (% of samples):", ", ".join(f"{n[6:]} {v:.1f}" for v, n in agg))
    print("  top instructions:")
    for r in sorted(data, key=lambda r: -num(r[ix[col]]))[:int(sys.argv[2]) if len(sys.argv) > 2 else 12]:
        smp = num(r[ix[col]])
        br = sorted(((num(r[ix[n]]), n[6:]) for n in stalls), reverse=True)[:2]
        print(f"    {smp / tot * 100:5.1f}%  {r[1][:58]:58s} {br}")
