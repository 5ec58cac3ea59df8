#!/bin/bash
# C3 tail-engine grid size and near-far delta sweep; FSteal ablation regression check (tail / swizzle)
O=gpurun_out/r16; mkdir -p $O
for cfg in "GUM_TAIL_CTAS_PER_SM=1" "GUM_TAIL_CTAS_PER_SM=2"; do
  env $cfg timeout 600 python bench.py --config C3 --steps 2 --warmup 2 --no-e2e --no-cpu > $O/c3.json 2>/dev/null
  python -c "import json; d=json.loads(open('$O/c3.json').read().strip().splitlines()[-1]); print('$cfg', d['value'], d['ms_per_step'])"
done
for dl in 2048 8192 16384; do
  timeout 600 python bench.py --config C3 --steps 2 --warmup 2 --no-e2e --no-cpu --sssp-delta $dl > $O/c3.json 2>/dev/null
  python -c "import json; d=json.loads(open('$O/c3.json').read().strip().splitlines()[-1]); print('delta $dl', d['value'], d['ms_per_step'])"
done
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --tail 8192 > $O/abl_t8192.txt 2>&1; cat $O/abl_t8192.txt
GUM_FILTER_SWIZZLE=0 timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 > $O/abl_sw0.txt 2>&1; cat $O/abl_sw0.txt
