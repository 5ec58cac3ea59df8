#!/bin/bash
# tail engine: CTA-buffered appends, speculative row/far loads -- parity + C3/C1/C2
O=gpurun_out/r15; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_next1.py -m gpu -q -x -k "tail or grid or near_far or hand or c1 or virtual or forced" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e --no-cpu > $O/bench_C3.json 2> $O/bench_C3.err
timeout 300 python bench.py --config C1 --steps 50 --no-cpu --no-e2e > $O/bench_C1.json 2> $O/bench_C1.err
timeout 400 python bench.py --no-cpu --no-e2e --no-variants > $O/bench_C2.json 2> $O/bench_C2.err
for f in C1 C2 C3; do python -c "import json; d=json.loads(open('$O/bench_$f.json').read().strip().splitlines()[-1]); r=d['roofline']; print('$f', d['value'], d['ms_per_step'], r['kernel'], r['frac'])"; done
