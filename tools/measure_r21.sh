#!/bin/bash
# BFS depths written by the filter: full GPU suite, C2 bench + profile + launch list, smoke
O=gpurun_out/r21; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
python __graft_entry__.py > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
timeout 400 python bench.py --no-cpu --no-e2e --no-variants > $O/bench_C2.json 2> $O/bench_C2.err
python -c "import json; d=json.loads(open('$O/bench_C2.json').read().strip().splitlines()[-1]); r=d['roofline']; print('C2', d['value'], d['ms_per_step'], r['frac'], d['detail']['parity_full_size'])"
python tools/profile_run.py --config C2 --alg bfs --runs 3 --part degree > $O/prof.txt 2>&1; tail -1 $O/prof.txt | cut -c1-200
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C2_bfs.csv python tools/profile_run.py --config C2 --alg bfs --runs 1 --part degree > /dev/null 2>&1
grep -E "k_advance|k_filter" $O/launches_C2_bfs.csv | awk -F'","' '{split($5,a,"("); printf "%s %.1f | ", substr(a[1],length(a[1])-8), $15/1000}'; echo
