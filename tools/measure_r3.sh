#!/bin/bash
# parity subset + C2 seg/degree bench and per-kernel profile (hub snapshot on/off)
O=gpurun_out/r3; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_next1.py -m gpu -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
for p in seg degree; do
  timeout 300 python bench.py --part $p > $O/bench_C2_$p.json 2> $O/bench_C2_$p.err; echo "C2 $p rc=$?"
  python tools/profile_run.py --config C2 --alg bfs --runs 3 --part $p > $O/prof_C2_$p.txt 2>&1
done
GUM_HUB_SNAP_WORDS=0 python tools/profile_run.py --config C2 --alg bfs --runs 3 --part degree > $O/prof_C2_degree_nosnap.txt 2>&1
GUM_HUB_SNAP_WORDS=2048 python tools/profile_run.py --config C2 --alg bfs --runs 3 --part degree > $O/prof_C2_degree_snap2k.txt 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C2_bfs_degree.csv python tools/profile_run.py --config C2 --alg bfs --runs 1 --part degree > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_advance -s 2 -c 1 -o $O/adv_C2_bfs_degree python tools/profile_run.py --config C2 --alg bfs --runs 1 --part degree > /dev/null 2>&1
echo done
