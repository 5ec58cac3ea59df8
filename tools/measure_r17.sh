#!/bin/bash
# P=8 virtual-worker regression check (session-start build vs now), C3 tail grid 3/4 CTAs per SM
O=gpurun_out/r17; mkdir -p $O
for lib in build/variants/libgum_old.so paper_conf_icde_menggltyz23_b200/libgum.so; do
  GUM_LIB=$lib python tools/profile_run.py --rmat 22 --noscramble --gpus 8 --runs 3 --alg bfs > $O/prof.txt 2>&1; echo "$lib"; tail -2 $O/prof.txt | cut -c1-400
done
for n in 3 4; do
  GUM_TAIL_CTAS_PER_SM=$n timeout 600 python bench.py --config C3 --steps 2 --warmup 2 --no-e2e --no-cpu > $O/c3.json 2>/dev/null
  python -c "import json; d=json.loads(open('$O/c3.json').read().strip().splitlines()[-1]); print('tail ctas $n', d['value'], d['ms_per_step'])"
done
