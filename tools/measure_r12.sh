#!/bin/bash
# tail default 16384: full GPU suite; C1/C2/C3 bench lines; tail 65536 on C3
O=gpurun_out/r12; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
timeout 400 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"
timeout 300 python bench.py --config C1 --steps 50 > $O/bench_C1.json 2> $O/bench_C1.err; echo "C1 rc=$?"
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e > $O/bench_C3.json 2> $O/bench_C3.err; echo "C3 rc=$?"
timeout 600 python bench.py --config C3 --steps 2 --warmup 3 --no-e2e --no-cpu --tail 65536 > $O/bench_C3_t65536.json 2> $O/bench_C3_t65536.err
for f in C1 C2 C3 C3_t65536; do python -c "import json; d=json.loads(open('$O/bench_$f.json').read().strip().splitlines()[-1]); print('$f', d['value'], d['ms_per_step'], d['roofline']['frac'], (d.get('detail') or {}).get('parity_full_size'))"; done
