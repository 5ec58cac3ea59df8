#!/bin/bash
# minimal shared-memory carveout for the advance by default: parity subset + C2..C5
O=gpurun_out/r25; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "virtual or hand or c1 or single_worker" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $O/pytest.log
python tools/profile_run.py --config C2 --alg bfs --runs 3 --part degree > $O/prof.txt 2>&1; tail -1 $O/prof.txt | cut -c1-150
timeout 400 python bench.py --no-cpu --no-e2e --no-variants > $O/bench_C2.json 2> $O/bench_C2.err
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e --no-cpu > $O/bench_C4.json 2> $O/bench_C4.err
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e --no-cpu > $O/bench_C5.json 2> $O/bench_C5.err
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e --no-cpu > $O/bench_C3.json 2> $O/bench_C3.err
for f in C2 C3 C4 C5; do python -c "import json; d=json.loads(open('$O/bench_$f.json').read().strip().splitlines()[-1]); r=d['roofline']; print('$f', d['value'], d['ms_per_step'], r['kernel'], r['frac'])"; done
