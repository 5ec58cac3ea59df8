#!/bin/bash
O=gpurun_out/r23; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_next1.py tests/test_gpu_mp.py -m gpu -q -x -k "bfs or c1 or relabel or hand or tail or mp" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
python tools/profile_run.py --config C2 --alg bfs --runs 3 --part degree > $O/prof.txt 2>&1; tail -1 $O/prof.txt | cut -c1-200
timeout 400 python bench.py --no-cpu --no-e2e --no-variants > $O/bench_C2.json 2> $O/bench_C2.err
python -c "import json; d=json.loads(open('$O/bench_C2.json').read().strip().splitlines()[-1]); r=d['roofline']; print('C2', d['value'], d['ms_per_step'], r['frac'])"
