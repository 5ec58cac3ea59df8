#!/bin/bash
# ncu --set full capture of the LONGEST launch of one kernel in a tools/profile_run.py run: a launch-list pass
# (gpu__time_duration of every launch) picks the launch index, then one full capture of that launch.
#   tools/ncu_longest.sh <out_dir> <kernel regex, e.g. k_tail> <profile_run.py args...>
O=$1; K=$2; shift 2; mkdir -p $O
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:$K --csv --log-file $O/list_$K.csv \
  python tools/profile_run.py "$@" > $O/list_$K.log 2>&1 || exit 1
idx=$(python - "$O/list_$K.csv" <<'PY'
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
s = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
h = rows[s]; vi = h.index("Metric Value")
vals = [float(r[vi].replace(",", "")) for r in rows[s + 1:]]
print(max(range(len(vals)), key=lambda i: vals[i]))
PY
)
echo "longest $K launch: index $idx"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s $idx -c 1 -o $O/full_$K -f \
  python tools/profile_run.py "$@" > $O/full_$K.log 2>&1
python tools/ncu_summary.py $O/full_$K.ncu-rep 14 > $O/ncu_full_$K.txt 2>&1; head -30 $O/ncu_full_$K.txt
