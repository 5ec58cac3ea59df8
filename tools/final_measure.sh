#!/bin/bash
# Final-state evidence run (one GPU): GPU tests, smoke, full-size parity of the configs whose path changed last
# (C3, C4), bench lines C2/C3/C4/C1, OSteal ablations, launch list + ncu of the C3 tail engine.
O=${O:-gpurun_out/fin}; mkdir -p $O
make -j4 all > $O/build.log 2>&1; echo "build rc=$?"
( time timeout 1800 python -m pytest tests -m gpu -q ) > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -4 $O/pytest.log | head -1
timeout 600 python __graft_entry__.py > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1800 python tools/parity_full.py --configs C3,C4 --out $O > $O/parity.log 2>&1; echo "parity rc=$?"
O=$O CONFIGS="${CONFIGS:-C2 C3 C4 C1}" bash tools/measure.sh
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --out $O/abl_osteal_virtual.json > $O/abl_osteal_virtual.txt 2>&1; cat $O/abl_osteal_virtual.txt
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --split --out $O/abl_osteal_split.json > $O/abl_osteal_split.txt 2>&1; cat $O/abl_osteal_split.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C3_sssp.csv \
  python tools/profile_run.py --config C3 --alg sssp --runs 1 > $O/launches_C3.log 2>&1; python tools/launches.py $O/launches_C3_sssp.csv > $O/launches_C3_sssp_summary.txt; head -8 $O/launches_C3_sssp_summary.txt
bash tools/ncu_longest.sh $O/ncu_tail k_tail 150 20 --config C3 --alg sssp --runs 1; rm -f $O/ncu_tail/*.ncu-rep
