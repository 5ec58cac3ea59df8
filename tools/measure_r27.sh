#!/bin/bash
O=gpurun_out/r27; mkdir -p $O
for t in 0 1024 4096 16384; do
  timeout 400 python bench.py --no-cpu --no-e2e --no-variants --tail $t > $O/c2_t$t.json 2>/dev/null
  python -c "import json; d=json.loads(open('$O/c2_t$t.json').read().strip().splitlines()[-1]); print('C2 tail $t', d['value'], d['ms_per_step'])"
done
for t in 0 4096 16384; do
  timeout 300 python bench.py --config C1 --steps 50 --no-cpu --no-e2e --no-variants --tail $t > $O/c1_t$t.json 2>/dev/null
  python -c "import json; d=json.loads(open('$O/c1_t$t.json').read().strip().splitlines()[-1]); print('C1 tail $t', d['value'], d['ms_per_step'])"
done
