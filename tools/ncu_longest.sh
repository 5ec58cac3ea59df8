#!/bin/bash
# ncu --set full capture of a long launch of one kernel in a tools/profile_run.py run whose launch sequence is
# not reproducible (the tail engine's entries depend on timing): capture a window of consecutive launches,
# then summarise the longest one of the window.
#   tools/ncu_longest.sh <out_dir> <kernel regex> <skip> <count> <profile_run.py args...>
O=$1; K=$2; S=$3; N=$4; shift 4; mkdir -p $O
timeout 1800 ncu --set full --clock-control none --import-source on -k regex:$K -s $S -c $N -o $O/full_$K -f \
  python tools/profile_run.py "$@" > $O/full_$K.log 2>&1
j=$(ncu -i $O/full_$K.ncu-rep --page raw --csv --metrics gpu__time_duration.sum 2>/dev/null | python -c "
import csv, sys
rows = list(csv.reader(sys.stdin))
h = rows[0]; i = h.index('gpu__time_duration.sum')
v = [float(r[i].replace(',', '')) for r in rows[2:]]
print(max(range(len(v)), key=lambda k: v[k]))")
echo "longest of the window: launch $j"
NCU_IMPORT_ARGS="--launch-skip $j --launch-count 1" python tools/ncu_summary.py $O/full_$K.ncu-rep 14 > $O/ncu_full_$K.txt 2>&1
head -30 $O/ncu_full_$K.txt
