#!/bin/bash
# re-measure the bench lines changed after tools/round_measure_final.sh (carveout, BFS tail default, tail engine)
O=gpurun_out/final2; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $O/pytest.log
python __graft_entry__.py > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 400 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"
timeout 300 python bench.py --config C1 --steps 50 > $O/bench_C1.json 2> $O/bench_C1.err; echo "C1 rc=$?"
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e > $O/bench_C3.json 2> $O/bench_C3.err; echo "C3 rc=$?"
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e > $O/bench_C4.json 2> $O/bench_C4.err; echo "C4 rc=$?"
for f in C1 C2 C3 C4; do python -c "import json; d=json.loads(open('$O/bench_$f.json').read().strip().splitlines()[-1]); r=d['roofline']; print('$f', d['value'], d['ms_per_step'], r['kernel'], r['frac'], (d.get('detail') or {}).get('parity_full_size',{}).get('exact'), d['e2e'] and round(d['e2e']['value'],2))"; done
P="python tools/profile_run.py --runs 1"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C2_bfs.csv $P --config C2 --alg bfs --part degree > /dev/null 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_advance --csv --log-file $O/traffic_C2_bfs.csv $P --config C2 --alg bfs --part degree > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_advance -s 3 -c 1 -o $O/adv_C2_bfs $P --config C2 --alg bfs --part degree > /dev/null 2>&1
echo done
