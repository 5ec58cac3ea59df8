#!/bin/bash
# Round-2 evidence run (one GPU): GPU tests, smoke, full-size parity, bench lines of every config, ablations,
# ncu launch list + captures. Outputs under $O (default gpurun_out/r2m); the summaries are copied to profiles/round2.
O=${O:-gpurun_out/r2m}; mkdir -p $O
make -j4 all > $O/build.log 2>&1; echo "build rc=$?"
( time timeout 1800 python -m pytest tests -m gpu -q ) > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -4 $O/pytest.log | head -1
timeout 600 python __graft_entry__.py > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1800 python tools/parity_full.py --configs C3,C4,C5 --out $O > $O/parity.log 2>&1; echo "parity rc=$?"
O=$O CONFIGS="${CONFIGS:-C2 C1 C3 C4 C5 C5:dpr}" bash tools/measure.sh
timeout 900 python tools/ablation.py --table4 --scale 22 --grid 2048 --workers 8 --delta 1024 --out $O/abl_table4.json > $O/abl_table4.txt 2>&1; echo "table4 rc=$?"; cat $O/abl_table4.txt
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --out $O/abl_fsteal_virtual.json > $O/abl_fsteal_virtual.txt 2>&1; cat $O/abl_fsteal_virtual.txt
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --split --out $O/abl_fsteal_split.json > $O/abl_fsteal_split.txt 2>&1; cat $O/abl_fsteal_split.txt
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --out $O/abl_osteal_virtual.json > $O/abl_osteal_virtual.txt 2>&1; cat $O/abl_osteal_virtual.txt
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --split --out $O/abl_osteal_split.json > $O/abl_osteal_split.txt 2>&1; cat $O/abl_osteal_split.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C2_bfs.csv \
  python tools/profile_run.py --config C2 --alg bfs --part degree --runs 1 > $O/launches_C2.log 2>&1; python tools/launches.py $O/launches_C2_bfs.csv > $O/launches_C2_bfs_summary.txt; head -12 $O/launches_C2_bfs_summary.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_advance -s 3 -c 1 -o $O/adv_C2 -f \
  python tools/profile_run.py --config C2 --alg bfs --part degree --runs 1 > $O/ncu_adv_C2.log 2>&1; python tools/ncu_summary.py $O/adv_C2.ncu-rep 12 > $O/ncu_full_k_advance_C2_bfs_peak.txt 2>&1; head -25 $O/ncu_full_k_advance_C2_bfs_peak.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pr_pull -s 14 -c 1 -o $O/pull_C5 -f \
  python tools/profile_run.py --config C5 --alg pr --part degree --runs 1 > $O/ncu_pull_C5.log 2>&1; python tools/ncu_summary.py $O/pull_C5.ncu-rep 12 > $O/ncu_full_k_pr_pull_C5.txt 2>&1; head -25 $O/ncu_full_k_pr_pull_C5.txt
timeout 900 python tools/ablation.py --next1 --scale 20 --workers 8 --out $O/abl_next1.json > $O/abl_next1.txt 2>&1; cat $O/abl_next1.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C3_sssp.csv \
  python tools/profile_run.py --config C3 --alg sssp --runs 1 > $O/launches_C3.log 2>&1; python tools/launches.py $O/launches_C3_sssp.csv > $O/launches_C3_sssp_summary.txt; head -8 $O/launches_C3_sssp_summary.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tail -s 5 -c 1 -o $O/tail_C3 -f \
  python tools/profile_run.py --config C3 --alg sssp --runs 1 > $O/ncu_tail_C3.log 2>&1; python tools/ncu_summary.py $O/tail_C3.ncu-rep 12 > $O/ncu_full_k_tail_C3_sssp.txt 2>&1; head -25 $O/ncu_full_k_tail_C3_sssp.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C5_pr.csv \
  python tools/profile_run.py --config C5 --alg pr --part degree --runs 1 > $O/launches_C5.log 2>&1; python tools/launches.py $O/launches_C5_pr.csv > $O/launches_C5_pr_summary.txt; head -8 $O/launches_C5_pr_summary.txt
