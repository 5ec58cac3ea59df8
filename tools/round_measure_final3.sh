#!/bin/bash
# re-measure after the fused dense filter tile: bench lines C2/C1/C4/C5, C2 launch list, ncu --set full of the C2 peak filter
O=gpurun_out/final3; mkdir -p $O
python __graft_entry__.py > $O/smoke.log 2>&1; echo "smoke rc=$?"
timeout 400 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"
timeout 300 python bench.py --config C1 --steps 50 > $O/bench_C1.json 2> $O/bench_C1.err; echo "C1 rc=$?"
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e > $O/bench_C4.json 2> $O/bench_C4.err; echo "C4 rc=$?"
for f in C1 C2 C4; do python -c "import json; d=json.loads(open('$O/bench_$f.json').read().strip().splitlines()[-1]); r=d['roofline']; print('$f', d['value'], d['ms_per_step'], r['kernel'], r['frac'], (d.get('detail') or {}).get('parity_full_size',{}).get('exact'), d['e2e'] and round(d['e2e']['value'],2))"; done
P="python tools/profile_run.py --runs 1"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_C2_bfs.csv $P --config C2 --alg bfs --part degree > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_filter -s 2 -c 1 -o $O/filt_C2_bfs $P --config C2 --alg bfs --part degree > /dev/null 2>&1
echo "ncu done"
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e > $O/bench_C5.json 2> $O/bench_C5.err; echo "C5 rc=$?"
python -c "import json; d=json.loads(open('$O/bench_C5.json').read().strip().splitlines()[-1]); r=d['roofline']; print('C5', d['value'], d['ms_per_step'], r['kernel'], r['frac'])"
