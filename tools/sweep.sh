#!/bin/bash
# usage: tools/sweep.sh "ENV1=a ENV2=b" "ENV1=c" ...   -- one profile_run per setting, per-kernel totals
for cfg in "$@"; do
  echo "== $cfg"
  env $cfg timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file /tmp/l.csv python tools/profile_run.py ${PR_ARGS:---config C2 --alg bfs --runs 1} > /dev/null 2>&1
  python tools/launches.py /tmp/l.csv 2>/dev/null | head -2
done
