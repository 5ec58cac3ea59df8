#!/bin/bash
O=gpurun_out/r22; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
timeout 400 python bench.py --no-cpu --no-e2e --no-variants > $O/bench_C2.json 2> $O/bench_C2.err
python tools/profile_run.py --config C2 --alg bfs --runs 3 --part degree > $O/prof.txt 2>&1; tail -1 $O/prof.txt | cut -c1-200
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e --no-cpu > $O/bench_C3.json 2> $O/bench_C3.err
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e --no-cpu > $O/bench_C4.json 2> $O/bench_C4.err
for f in C2 C3 C4; do python -c "import json; d=json.loads(open('$O/bench_$f.json').read().strip().splitlines()[-1]); r=d['roofline']; print('$f', d['value'], d['ms_per_step'], r['kernel'], r['frac'])"; done
