#!/bin/bash
# tail engine: whole-warp path for >32-edge lists, 3 CTAs/SM; parity + P=8 profile + C1/C2/C3
O=gpurun_out/r18; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_next1.py -m gpu -q -x -k "tail or grid or near_far or hand or c1 or virtual or forced or stealing" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
python tools/profile_run.py --rmat 22 --noscramble --gpus 8 --runs 3 --alg bfs > $O/prof.txt 2>&1; tail -1 $O/prof.txt | cut -c1-300
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e --no-cpu > $O/bench_C3.json 2> $O/bench_C3.err
timeout 300 python bench.py --config C1 --steps 50 --no-cpu --no-e2e > $O/bench_C1.json 2> $O/bench_C1.err
timeout 400 python bench.py --no-cpu --no-e2e --no-variants > $O/bench_C2.json 2> $O/bench_C2.err
for f in C1 C2 C3; do python -c "import json; d=json.loads(open('$O/bench_$f.json').read().strip().splitlines()[-1]); r=d['roofline']; print('$f', d['value'], d['ms_per_step'], r['kernel'], r['frac'])"; done
timeout 600 python tools/ablation.py --fsteal --scale 22 --workers 8 --out $O/abl_fsteal_virtual.json > $O/abl_fsteal.txt 2>&1; cat $O/abl_fsteal.txt
