#!/bin/bash
# relabel fix check, e2e breakdown, C3 tail-threshold sweep, C5 PR block-size / occupancy sweep
O=gpurun_out/r11; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "relabel or invariance or c1 or single_worker" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
timeout 400 python bench.py --no-cpu --no-variants > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"
python -c "import json; d=json.loads(open('$O/bench_C2.json').read().strip().splitlines()[-1]); print(d['value'], d['e2e'])"
for t in 16384 32768; do
  timeout 600 python bench.py --config C3 --steps 2 --warmup 3 --no-e2e --no-cpu --tail $t > $O/bench_C3_t$t.json 2> $O/bench_C3_t$t.err
  python -c "import json; d=json.loads(open('$O/bench_C3_t$t.json').read().strip().splitlines()[-1]); print('C3 tail $t', d['value'], d['ms_per_step'])"
done
for bb in 33554432 67108864; do
  GUM_PR_BLOCK_BYTES=$bb timeout 600 python bench.py --config C5 --steps 2 --warmup 3 --no-e2e --no-cpu > $O/bench_C5_b$bb.json 2> $O/bench_C5_b$bb.err
  python -c "import json; d=json.loads(open('$O/bench_C5_b$bb.json').read().strip().splitlines()[-1]); print('C5 block $bb', d['value'], d['ms_per_step'])"
done
GUM_ADV_CTAS_PER_SM=3 timeout 600 python bench.py --config C5 --steps 2 --warmup 3 --no-e2e --no-cpu > $O/bench_C5_occ3.json 2> $O/bench_C5_occ3.err
python -c "import json; d=json.loads(open('$O/bench_C5_occ3.json').read().strip().splitlines()[-1]); print('C5 occ3', d['value'], d['ms_per_step'])"
