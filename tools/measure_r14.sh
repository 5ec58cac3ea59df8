#!/bin/bash
# round measurement refresh (all configs with CPU baseline and e2e), launch lists, ncu of C3 tail and C5 PR
O=gpurun_out/r14; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
timeout 400 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"
timeout 300 python bench.py --config C1 --steps 50 > $O/bench_C1.json 2> $O/bench_C1.err; echo "C1 rc=$?"
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e > $O/bench_C3.json 2> $O/bench_C3.err; echo "C3 rc=$?"
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e > $O/bench_C4.json 2> $O/bench_C4.err; echo "C4 rc=$?"
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e > $O/bench_C5.json 2> $O/bench_C5.err; echo "C5 rc=$?"
timeout 600 python bench.py --impl reference --steps 3 > $O/bench_ref_C2.json 2> $O/bench_ref_C2.err; echo "ref rc=$?"
for f in C1 C2 C3 C4 C5; do python -c "import json; d=json.loads(open('$O/bench_$f.json').read().strip().splitlines()[-1]); r=d['roofline']; print('$f', d['value'], d['ms_per_step'], r['kernel'], r['frac'], (d.get('detail') or {}).get('parity_full_size',{}).get('exact'), d['e2e'] and round(d['e2e']['value'],2))"; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C2_bfs.csv python tools/profile_run.py --config C2 --alg bfs --runs 1 --part degree > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C5_pr.csv python tools/profile_run.py --config C5 --alg pr --runs 1 > /dev/null 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_advance --csv --log-file $O/traffic_C5_pr.csv python tools/profile_run.py --config C5 --alg pr --runs 1 > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_advance -s 10 -c 1 -o $O/adv_C5_pr python tools/profile_run.py --config C5 --alg pr --runs 1 > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_tail -s 40 -c 1 -o $O/tail_C3_sssp python tools/profile_run.py --config C3 --alg sssp --runs 1 > /dev/null 2>&1
echo "ncu done"
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --out $O/abl_fsteal_virtual.json > $O/abl_fsteal.txt 2>&1
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --out $O/abl_osteal_virtual.json > $O/abl_osteal.txt 2>&1
echo done
