#!/bin/bash
O=gpurun_out/r8; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "pr" > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $O/pytest.log
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e --no-cpu > $O/bench_C5.json 2> $O/bench_C5.err; echo "C5 rc=$?"; tail -c 250 $O/bench_C5.json
GUM_PR_PUSH=0 timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e --no-cpu > $O/bench_C5_adv.json 2> $O/bench_C5_adv.err; echo "C5 adv rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_pr_push -s 5 -c 1 -o $O/push_C5_pr python tools/profile_run.py --config C5 --alg pr --runs 1 > /dev/null 2>&1; echo "ncu rc=$?"
