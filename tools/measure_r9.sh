#!/bin/bash
# warp-independent filter pass 2: full GPU suite, C2/C3/C4 bench, C2 per-kernel profile
O=gpurun_out/r9; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $O/pytest.log
timeout 400 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err; echo "C2 rc=$?"; tail -c 200 $O/bench_C2.json
python tools/profile_run.py --config C2 --alg bfs --runs 3 --part degree > $O/prof_C2.txt 2>&1; tail -1 $O/prof_C2.txt
timeout 900 python bench.py --config C4 --steps 5 --warmup 3 --no-e2e --no-cpu > $O/bench_C4.json 2> $O/bench_C4.err; echo "C4 rc=$?"; tail -c 200 $O/bench_C4.json
timeout 900 python bench.py --config C3 --steps 3 --warmup 3 --no-e2e --no-cpu > $O/bench_C3.json 2> $O/bench_C3.err; echo "C3 rc=$?"; tail -c 200 $O/bench_C3.json
