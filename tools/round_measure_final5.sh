#!/bin/bash
# bench lines at HEAD after the packed tile scan: C2 (default), C1, C4
O=gpurun_out/final5; mkdir -p $O
timeout 400 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"
timeout 300 python bench.py --config C1 --steps 50 > $O/bench_C1.json 2> $O/bench_C1.err; echo "C1 rc=$?"
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e > $O/bench_C4.json 2> $O/bench_C4.err; echo "C4 rc=$?"
for f in C1 C2 C4; do python -c "import json; d=json.loads(open('$O/bench_$f.json').read().strip().splitlines()[-1]); r=d['roofline']; print('$f', d['value'], d['ms_per_step'], r['kernel'], r['achieved'], r['frac'], (d.get('detail') or {}).get('parity_full_size',{}).get('exact'), d['e2e'] and round(d['e2e']['value'],2), d['cpu_baseline']['value'], d['clocks'])"; done
