#!/bin/bash
# shared-memory carveout hint for the advance (L1 capacity for the visited-bit probes), C2
O=gpurun_out/r24; mkdir -p $O
for cv in -1 35 45 60 100; do
  GUM_SMEM_CARVEOUT=$cv python tools/profile_run.py --config C2 --alg bfs --runs 3 --part degree > $O/prof_$cv.txt 2>&1
  echo "carveout $cv $(tail -1 $O/prof_$cv.txt | cut -c1-110)"
done
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_next1.py tests/test_gpu_mp.py -m gpu -q -x -k "tail or grid or near_far or hand or virtual or forced or stealing or mp or mirrors" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
timeout 900 python tools/ablation.py --osteal --grid 2048 --workers 8 --delta 1024 --out $O/abl_osteal_virtual.json > $O/abl_osteal.txt 2>&1; cat $O/abl_osteal.txt
python tools/profile_run.py --rmat 22 --noscramble --gpus 8 --runs 3 --alg bfs > $O/prof8.txt 2>&1; tail -1 $O/prof8.txt | cut -c1-300
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e --no-cpu > $O/bench_C3.json 2> $O/bench_C3.err
python -c "import json; d=json.loads(open('$O/bench_C3.json').read().strip().splitlines()[-1]); r=d['roofline']; print('C3', d['value'], d['ms_per_step'], r['kernel'], r['frac'])"
