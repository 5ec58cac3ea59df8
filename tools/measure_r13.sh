#!/bin/bash
# BFS hub discovery dedupe (DEGREE layout): parity + C2 on/off
O=gpurun_out/r13; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_next1.py -m gpu -q -x -k "bfs or c1 or relabel" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
for hd in 1 0; do
  GUM_HUB_DEDUP=$hd python tools/profile_run.py --config C2 --alg bfs --runs 3 --part degree > $O/prof_hd$hd.txt 2>&1; echo "hd=$hd $(tail -1 $O/prof_hd$hd.txt | cut -c1-110)"
  GUM_HUB_DEDUP=$hd timeout 400 python bench.py --no-cpu --no-e2e --no-variants > $O/bench_C2_hd$hd.json 2> $O/bench_C2_hd$hd.err
  python -c "import json; d=json.loads(open('$O/bench_C2_hd$hd.json').read().strip().splitlines()[-1]); print('C2 hd=$hd', d['value'], d['ms_per_step'])"
done
GUM_HUB_DEDUP=1 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C2_bfs.csv python tools/profile_run.py --config C2 --alg bfs --runs 1 --part degree > /dev/null 2>&1
grep -E "k_advance" $O/launches_C2_bfs.csv | awk -F'","' '{printf "%.1f ", $15/1000}'; echo
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e --no-cpu > $O/bench_C3.json 2> $O/bench_C3.err
python -c "import json; d=json.loads(open('$O/bench_C3.json').read().strip().splitlines()[-1]); print('C3', d['value'], d['ms_per_step'], d['roofline'])"
