#!/bin/bash
O=gpurun_out/r30; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_next1.py -m gpu -q -x -k "tail or grid or near_far or hand or virtual" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $O/pytest.log
for n in 2 3; do
  GUM_TAIL_CTAS_PER_SM=$n python tools/profile_run.py --grid 2048 --alg sssp --gpus 8 --delta 1024 --osteal-threshold 4096 --runs 2 > $O/prof_$n.txt 2>&1; echo "P8 grid tail ctas $n $(tail -1 $O/prof_$n.txt | cut -c1-200)"
  GUM_TAIL_CTAS_PER_SM=$n timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e --no-cpu > $O/c3_$n.json 2>/dev/null
  python -c "import json; d=json.loads(open('$O/c3_$n.json').read().strip().splitlines()[-1]); print('C3 tail ctas $n', d['value'], d['ms_per_step'])"
done
