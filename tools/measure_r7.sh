#!/bin/bash
# grouped tail engine phase 1 + PR warp-task push: parity, C3/C5/C1 bench
O=gpurun_out/r7; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-e2e > $O/bench_C5.json 2> $O/bench_C5.err; echo "C5 rc=$?"; tail -c 250 $O/bench_C5.json
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e > $O/bench_C3.json 2> $O/bench_C3.err; echo "C3 rc=$?"; tail -c 250 $O/bench_C3.json
timeout 300 python bench.py --config C1 --steps 50 > $O/bench_C1.json 2> $O/bench_C1.err; echo "C1 rc=$?"; tail -c 250 $O/bench_C1.json
timeout 400 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"; tail -c 250 $O/bench_C2.json
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_pr_push -s 5 -c 1 -o $O/push_C5_pr python tools/profile_run.py --config C5 --alg pr --runs 1 > /dev/null 2>&1; echo "ncu rc=$?"
echo done
